F=gpurun_out/r3o; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
PAGODA_CE_STATS=1 timeout 200 python bench.py --workload mm --quick --no-configs > $F/mm.json 2> $F/mm_ce_stats.txt
grep "pagoda CE" $F/mm_ce_stats.txt | tail -5
PAGODA_CE_STATS=1 timeout 200 python bench.py --workload mm --quick --no-configs --prespawn > $F/mmpre.json 2> $F/mmpre_ce_stats.txt
grep "pagoda CE" $F/mmpre_ce_stats.txt | tail -3
timeout 300 python scripts/probe_life.py mm > $F/life.jsonl 2> $F/life.err; cat $F/life.jsonl
DRAIN=1 timeout 300 python scripts/probe_life.py mm > $F/life_drain.jsonl 2>> $F/life.err; cat $F/life_drain.jsonl
tail -2 $F/life.err
