# A/B of the wide cooperative refine: the previous build, then the new builds at several
# GSWORD_OPT_COOP_WIDE thresholds (option 17).
set -u
mkdir -p gpurun_out
W=${VB_WORK:-C1:1,C1:2,C1:0,C2:0,C3:0}
VB_WORK=$W python scripts/variant_bench.py build/variants/lib_a_base.so > gpurun_out/abw.jsonl 2> gpurun_out/abw.err
for T in -1 4096 1024 256; do
  VB_WORK=$W VB_OPTS=17=$T VB_TAG=":wide$T" python scripts/variant_bench.py build/variants/lib_h_wide4.so >> gpurun_out/abw.jsonl 2>> gpurun_out/abw.err
done
for T in 1024 256; do
  VB_WORK=$W VB_OPTS=17=$T VB_TAG=":wide$T" python scripts/variant_bench.py build/variants/lib_i_wide2.so >> gpurun_out/abw.jsonl 2>> gpurun_out/abw.err
done
echo done
