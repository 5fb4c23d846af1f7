timeout 300 python scripts/probe_session_overhead.py > gpurun_out/session_overhead.json 2>&1; cat gpurun_out/session_overhead.json
for r in 1 2 3; do for v in 0 mbilp; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 300 python bench.py --workload mb --quick --no-cpu --no-naive --steps 10 2>/dev/null | tail -1 > gpurun_out/ab6_mb_${v}_$r.json
  echo "$v $r $(python -c "import json;d=json.load(open('gpurun_out/ab6_mb_${v}_$r.json'));print(round(d['value']/1e6,3), d['ms_per_step'])")"
done; done
export PAGODA_LIB=$PWD/build/variants/libpagoda_vmbilp.so
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "mandelbrot or naive or fusion" 2>&1 | tail -1
