export PAGODA_LIB=$PWD/build/variants/libpagoda_vfast.so
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_runtime.py tests/test_gpu_workloads.py -q -x -k "not full_size" 2>&1 | tail -1
for r in 1 2; do for v in 0 fast fast2; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  line="$v $r"
  for w in tdes mm nop mb mix; do
    timeout 300 python bench.py --workload $w --quick --no-cpu --no-naive --steps 5 2>/dev/null | tail -1 > gpurun_out/ab8_${w}_${v}_$r.json
    line="$line $w=$(python -c "import json;d=json.load(open('gpurun_out/ab8_${w}_${v}_$r.json'));print(round(d['value']/1e6,2))")"
  done
  echo $line
done; done
export PAGODA_LIB=$PWD/build/variants/libpagoda_vfastp.so
timeout 300 python scripts/probe_prof.py > gpurun_out/prof_fast.json 2>&1
