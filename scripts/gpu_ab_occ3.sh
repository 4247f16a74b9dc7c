# A/B of occupancy variant 3 (wide cooperative rounds): previous build; new build autotuned,
# forced 1 (same occupancy, one-chunk rounds) and forced 3.
set -u
mkdir -p gpurun_out
W=${VB_WORK:-C1:1,C1:2,C1:0,C2:0,C3:0}
VB_WORK=$W python scripts/variant_bench.py build/variants/lib_a_base.so > gpurun_out/ab3.jsonl 2> gpurun_out/ab3.err
for O in -1 1 3; do
  VB_WORK=$W VB_OPTS=14=$O VB_TAG=":occ$O" python scripts/variant_bench.py build/variants/lib_j_occ3.so >> gpurun_out/ab3.jsonl 2>> gpurun_out/ab3.err
done
echo done
