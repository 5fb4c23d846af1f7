F=gpurun_out/r2d; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh hp "-DPAGODA_HOLDER_POSTS=1" hpc "-DPAGODA_HOLDER_POSTS=1 -DPAGODA_CTA_FENCE=1" \
  hpl "-DPAGODA_HOLDER_POSTS=1 -DPAGODA_LOOKAHEAD=2 -DPAGODA_CLAIM_SMALL=2" > $F/variants.log 2>&1
VARS="0 hp hpc hpl" AB=r2d TESTS=1 bash scripts/gpu_ab.sh
