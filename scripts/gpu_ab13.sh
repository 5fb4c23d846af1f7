for r in 1 2; do for v in 0 i256 i64; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  lat=$(timeout 300 python scripts/probe_latency.py 2>&1 | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print('iso',round(d['isolated_nop128_us']['p50'],2),'tdes',round(d['loaded_tdes_us']['p50'],1),'mix',round(d['loaded_mix_us']['p50'],1))")
  line="$v $r $lat"
  for w in tdes nop mm; do line="$line $w=$(timeout 300 python bench.py --workload $w --quick --no-cpu --no-naive 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']/1e6,2))")"; done
  echo $line
done; done
