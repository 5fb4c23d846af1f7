F=gpurun_out/r2e; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh prof "-DPAGODA_PROFILE=1" hpl "-DPAGODA_LOOKAHEAD=2 -DPAGODA_CLAIM_SMALL=2" lk3 "-DPAGODA_LOOKAHEAD=3 -DPAGODA_CLAIM_SMALL=4 -DPAGODA_SMALL_MULT=1" > $F/variants.log 2>&1
timeout 300 python scripts/probe_sched.py mm nop tdes > $F/sched.jsonl 2> $F/sched.err
PAGODA_LIB=build/variants/libpagoda_vprof.so timeout 300 python scripts/probe_prof.py > $F/prof.jsonl 2> $F/prof.err
VARS="0 hpl lk3" AB=r2e ABW="mm nop tdes" bash scripts/gpu_ab.sh > $F/ab.txt 2>&1
cat $F/ab.txt
