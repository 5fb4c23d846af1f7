# every benchmark body as a call (bni) vs 3DES / MM / MM64 / DCT only (0)
F=gpurun_out/r4f; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh bni "-DPAGODA_BODIES_NOINLINE=1" > $F/variants.log 2>&1
for i in 1 2; do for v in 0 bni; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  for w in tdes mm mb mix mpe mm_tc; do timeout 200 python bench.py --workload $w --quick --no-configs 2>/dev/null | tail -1 > $F/${w}_$v\_$i.json; done
  timeout 300 python bench.py --workload c5 --quick --no-configs --steps 3 --warmup 1 2>/dev/null | tail -1 > $F/c5_$v\_$i.json
done; done
unset PAGODA_LIB
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
