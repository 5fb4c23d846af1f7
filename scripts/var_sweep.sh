for v in ${VARS:-0 1 2 3 4 5}; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/exp_variants/libpagoda_v$v.so; fi
  timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "tdes and not naive" 2>&1 | tail -1 > gpurun_out/var_t$v.txt
  for i in 1 2; do timeout 300 python bench.py --workload tdes --quick --no-cpu --no-naive 2>/dev/null | tail -1 > gpurun_out/var_b${v}_$i.json; done
done
