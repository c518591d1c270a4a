#!/bin/bash
# compute-sanitizer over tools/sanitize_driver.py (every kernel family on tiny graphs), one log per tool.
# usage: tools/sanitize.sh [OUTDIR]     exit code: number of tools that reported errors
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
fails=0
for tool in memcheck racecheck synccheck initcheck; do
    extra=""
    [ "$tool" = "memcheck" ] && extra="--leak-check no"
    [ "$tool" = "initcheck" ] && extra=""
    timeout 900 compute-sanitizer --tool $tool $extra --error-exitcode 9 --print-limit 20 \
        python tools/sanitize_driver.py > "$OUT/sanitize_$tool.log" 2>&1
    rc=$?
    echo "$tool rc=$rc $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' "$OUT/sanitize_$tool.log" | tail -1)"
    [ $rc -ne 0 ] && fails=$((fails + 1))
done
exit $fails
