# Cooperative-refine threshold sweep on the final build (autotuned occupancy)
set -u
mkdir -p gpurun_out
W=${VB_WORK:-C1:1,C1:2,C2:0}
for T in 32 48 64 96 128; do
  VB_WORK=$W VB_OPTS=4=$T VB_TAG=":coop$T" python scripts/variant_bench.py build/variants/lib_u_head.so >> gpurun_out/coop.jsonl 2>> gpurun_out/coop.err
done
echo done
