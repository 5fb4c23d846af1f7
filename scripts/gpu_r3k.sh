# MM ncu capture (doorbell ingest at the preset's 24 KiB arena) and more host producers
F=gpurun_out/r3k; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
for i in 1 2; do for pr in 3 4 6; do
  timeout 200 python bench.py --workload mm --quick --no-configs --producers $pr 2>/dev/null | tail -1 > $F/mm_p${pr}_$i.json
done; done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:master_kernel -c 1 -o $F/ncu_mm python bench.py --workload mm --quick --no-configs --prespawn --steps 1 --warmup 0 --ce 0 > $F/ncu_mm_run.log 2>&1
python scripts/ncu_summary.py $F/ncu_mm.ncu-rep > $F/ncu_mm_full.txt 2>&1; head -3 $F/ncu_mm_full.txt
