# Is MM arrival-bound (host spawn / ingest) or MTB-bound?  producers 1/2/3 and a prespawned drain
F=gpurun_out/r2t; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
for i in 1 2; do
  for pr in 1 2 3; do timeout 200 python bench.py --workload mm --quick --no-configs --producers $pr 2>/dev/null | tail -1 > $F/mm_p$pr\_$i.json; done
  timeout 200 python bench.py --workload mm --quick --no-configs --prespawn 2>/dev/null | tail -1 > $F/mm_pre_$i.json
  timeout 200 python bench.py --workload tdes --quick --no-configs --prespawn 2>/dev/null | tail -1 > $F/tdes_pre_$i.json
  timeout 200 python bench.py --workload nop --quick --no-configs --prespawn 2>/dev/null | tail -1 > $F/nop_pre_$i.json
done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
