# 3DES body as a call (tni) vs inlined into the executor
F=gpurun_out/r4d; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh tni "-DPAGODA_TDES_NOINLINE=1" > $F/variants.log 2>&1
for i in 1 2 3; do for v in 0 tni; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 200 python bench.py --workload tdes --quick --no-configs 2>/dev/null | tail -1 > $F/tdes_$v\_$i.json
done; done
unset PAGODA_LIB
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
