# CE copies in flight (3 / 6); mix with 2 producers + the open-loop Poisson latency variant (C4)
F=gpurun_out/r3n; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh if6 "-DPAGODA_CE_INFLIGHT=6" > $F/variants.log 2>&1
for i in 1 2; do for v in 0 if6; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 200 python bench.py --workload mm --quick --no-configs 2>/dev/null | tail -1 > $F/mm_$v\_$i.json
  timeout 200 python bench.py --workload nop --quick --no-configs 2>/dev/null | tail -1 > $F/nop_$v\_$i.json
done; done
unset PAGODA_LIB
timeout 600 python bench.py --workload mix --no-configs --no-e2e --no-cpu --no-naive > $F/mix_full.json 2> $F/mix_full.err
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
python -c "
import json; d=json.loads(open('$F/mix_full.json').read().strip().splitlines()[-1]); print(d['value']/1e6, json.dumps(d.get('latency'))[:900])"
tail -3 $F/mix_full.err
