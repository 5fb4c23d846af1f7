# completion forwarders at 4 MTBs/SM (MM preset: CE ingest leaves MTB 0's ingest warps idle)
F=gpurun_out/r3q; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh f2 "-DPAGODA_FWD_4MTB=2" f3 "-DPAGODA_FWD_4MTB=3" > $F/variants.log 2>&1
for i in 1 2; do for v in 0 f2 f3; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 200 python bench.py --workload mm --quick --no-configs 2>/dev/null | tail -1 > $F/mm_$v\_$i.json
  timeout 200 python bench.py --workload mm --quick --no-configs --prespawn 2>/dev/null | tail -1 > $F/mmpre_$v\_$i.json
done; done
unset PAGODA_LIB
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
