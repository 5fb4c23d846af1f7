export PAGODA_LIB=$PWD/build/variants/libpagoda_vpair.so
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "tdes" 2>&1 | tail -1
for r in 1 2 3; do for v in 0 pair; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 300 python bench.py --workload tdes --quick --no-cpu --no-naive --steps 10 2>/dev/null | tail -1 > gpurun_out/ab7_${v}_$r.json
  echo "$v $r $(python -c "import json;d=json.load(open('gpurun_out/ab7_${v}_$r.json'));print(round(d['value']/1e6,3), round(d['roofline']['frac'],3))")"
done; done
