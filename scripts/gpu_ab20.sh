# Loaded-latency A/B (full tdes line without baselines) + claim-order variants (quick benches).
O=gpurun_out/ab20; mkdir -p $O
for v in 0 fwd1 acq0; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  for i in 1 2; do
    timeout 300 python bench.py --no-naive --no-cpu --no-e2e 2>/dev/null | tail -1 > $O/lat_tdes_${v}_$i.json
    python -c "import json;d=json.loads(open('$O/lat_tdes_${v}_$i.json').read().strip().splitlines()[-1]);print('$v', round(d['value']/1e6,2), d['latency']['loaded_us'], d['latency']['isolated_nop128_us'])"
  done
done
unset PAGODA_LIB
VARS="0 cfl2 cfl1 l2" AB=ab20 bash scripts/gpu_ab.sh
