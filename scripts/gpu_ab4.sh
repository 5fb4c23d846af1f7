for v in p1 0 p4; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 300 python scripts/probe_runtime.py > gpurun_out/ab4_probe_$v.json 2>&1
  timeout 300 python bench.py --workload mm --prespawn --quick --no-cpu --no-naive --steps 3 2>/dev/null | tail -1 > gpurun_out/ab4_pre_mm_$v.json
done
