# 3DES FMA-pipe sum A/B; fixed pipe peaks; MM life cycle with 1/2 producers and the device-only drain
F=gpurun_out/r2c; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh xor "-DPAGODA_TDES_FMA_SUM=0" > $F/variants.log 2>&1
python -c "
from paper_conf_ppopp_yehsser17_b200 import pagoda as PG
print('lds', PG.pipe_peak(0,'lds')); print('int32', PG.pipe_peak(0,'int32'))" > $F/peaks.txt 2>&1
for i in 1 2; do
  timeout 300 python bench.py --quick --no-configs > $F/tdes_sum_$i.json 2>> $F/err.log
  PAGODA_LIB=build/variants/libpagoda_vxor.so timeout 300 python bench.py --quick --no-configs > $F/tdes_xor_$i.json 2>> $F/err.log
done
timeout 300 python scripts/probe_life.py mm > $F/life_mm_p1.jsonl 2>> $F/err.log
PRODUCERS=2 timeout 300 python scripts/probe_life.py mm > $F/life_mm_p2.jsonl 2>> $F/err.log
DRAIN=1 timeout 300 python scripts/probe_life.py mm nop > $F/life_drain.jsonl 2>> $F/err.log
for p in 2 3; do timeout 300 python bench.py --quick --no-configs --workload mm --producers $p > $F/mm_p$p.json 2>> $F/err.log; done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $F/launches_tdes.csv python bench.py --quick --no-configs --prespawn --steps 2 --warmup 1 > $F/ncu_launch_run.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:master_kernel -c 1 -o $F/ncu_tdes python bench.py --quick --no-configs --prespawn --steps 1 --warmup 0 > $F/ncu_full_run.log 2>&1
for f in $F/tdes_*.json $F/mm_p*.json; do python -c "import json,sys;d=json.loads(open('$f').read().strip().splitlines()[-1]);print('$f', round(d['value']/1e6,2), round(d['roofline']['frac'],3))"; done
cat $F/peaks.txt
