for r in 1 2; do for v in head 0 p1; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  echo "$v $r $(timeout 300 python scripts/probe_latency.py 2>&1 | tail -1)"
done; done
unset PAGODA_LIB
timeout 600 python -m pytest tests/test_gpu_runtime.py -q -x 2>&1 | tail -1
for w in tdes nop mm; do timeout 300 python bench.py --workload $w --quick --no-cpu --no-naive 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print('$w',round(d['value']/1e6,2))"; done
