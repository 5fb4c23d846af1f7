F=gpurun_out/r2j; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh prof "-DPAGODA_PROFILE=1" > $F/variants.log 2>&1
PAGODA_LIB=build/variants/libpagoda_vprof.so timeout 300 python scripts/probe_prof.py > $F/prof.jsonl 2> $F/prof.err
DRAIN=1 timeout 300 python scripts/probe_life.py tdes mm > $F/life.jsonl 2> $F/life.err
cat $F/prof.jsonl
