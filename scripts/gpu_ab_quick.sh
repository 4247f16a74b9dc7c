# Quick A/B of compile-time variants (no test suite): variant_bench over build/variants/*.so
set -u
mkdir -p gpurun_out
VB_WORK=${VB_WORK:-C1:1,C1:2,C1:0,C2:0,C3:0} timeout ${VB_TIMEOUT:-1500} python scripts/variant_bench.py ${AB_LIBS:-build/variants/*.so} > gpurun_out/ab_variants.jsonl 2> gpurun_out/ab_variants.err
echo done
