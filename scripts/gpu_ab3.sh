timeout 600 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_workloads.py -q -x -k "not full_size" 2>&1 | tail -1
for r in 1 2; do for v in base 0 p1 p2; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  for w in tdes mm nop; do
    timeout 300 python bench.py --workload $w --quick --no-cpu --no-naive 2>/dev/null | tail -1 > gpurun_out/ab3_${w}_${v}_$r.json
    python -c "import json;d=json.load(open('gpurun_out/ab3_${w}_${v}_$r.json'));print('$w $v $r',round(d['value']/1e6,2), round(d['host_tasks_per_s']/1e6,2))"
  done
done; done
unset PAGODA_LIB
timeout 300 python scripts/probe_busy.py mm tdes > gpurun_out/busy2.json 2>&1; cat gpurun_out/busy2.json
