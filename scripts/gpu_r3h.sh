# MM: smaller arenas leave L1 to the executors' register spills (the carveout follows shared memory);
# the copy-engine ingest needs no staging shared memory in MTB 0
F=gpurun_out/r3h; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
for i in 1 2; do
  for ak in 48 32 24 16; do
    timeout 200 python bench.py --workload mm --quick --no-configs --ce 1 --arena-kb $ak 2>/dev/null | tail -1 > $F/mmce_a${ak}_$i.json
  done
  for ak in 48 32; do
    timeout 200 python bench.py --workload mm --quick --no-configs --ce 0 --arena-kb $ak 2>/dev/null | tail -1 > $F/mmdb_a${ak}_$i.json
  done
  timeout 200 python bench.py --workload mm --quick --no-configs --ce 1 --arena-kb 16 --prespawn 2>/dev/null | tail -1 > $F/mmcepre_a16_$i.json
  timeout 200 python bench.py --workload nop --quick --no-configs --ce 1 --arena-kb 16 2>/dev/null | tail -1 > $F/nopce_a16_$i.json
  timeout 200 python bench.py --workload mix --quick --no-configs --ce 1 2>/dev/null | tail -1 > $F/mixce_a200_$i.json
done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
