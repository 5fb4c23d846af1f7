F=gpurun_out/r3w; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh nfp "-DPAGODA_FREE_BEFORE_POST=0" ndi "-DPAGODA_DIRECT_IDLE_NS=0" > $F/variants.log 2>&1
for v in 0 nfp ndi; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 150 python bench.py --workload mb --quick --no-configs --max-tasks 1 > $F/out_$v.txt 2>&1; echo "$v rc=$?"
  timeout 150 python bench.py --workload tdes --quick --no-configs --max-tasks 1 > $F/outt_$v.txt 2>&1; echo "$v tdes rc=$?"
done
