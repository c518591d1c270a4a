LIB=paper_conf_eurosys_wumcjlzcy21_b200/libseastar.so
cp $LIB /tmp/orig.so
for v in mb0 mb6 mb0 mb6; do cp variants/libseastar_$v.so $LIB; echo -n "$v "; python bench.py --model gcn --steps 20 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],3), {k: round(v['ms'],3) for k,v in d['kernels'].items()})"; done
cp /tmp/orig.so $LIB
