# A/B of library variants: VARS="0 2 3" bash scripts/var_ab.sh  (0 = the in-tree build)
mkdir -p gpurun_out
for v in ${VARS:-0}; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 400 python -m pytest tests/test_gpu_parity.py tests/test_gpu_runtime.py -q -x -k "not full_size" 2>&1 | tail -1 > gpurun_out/ab_t$v.txt
  for w in ${ABW:-tdes mm}; do for i in 1 2; do
    timeout 300 python bench.py --workload $w --quick --no-cpu --no-naive 2>/dev/null | tail -1 > gpurun_out/ab_${w}_${v}_$i.json
  done; done
  timeout 300 python scripts/probe_runtime.py > gpurun_out/ab_probe_$v.json 2>&1
done
