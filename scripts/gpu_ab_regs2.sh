# A/B: register-pressure changes with and without the split edge-set probe, occupancy 0/2 and autotuned
set -u
mkdir -p gpurun_out
W=${VB_WORK:-C1:1,C1:2,C1:0}
VB_WORK=$W python scripts/variant_bench.py build/variants/lib_a_base.so > gpurun_out/abr2.jsonl 2> gpurun_out/abr2.err
for O in -1 0 2; do
  VB_WORK=$W VB_OPTS=14=$O VB_TAG=":occ$O" python scripts/variant_bench.py build/variants/lib_n_regs.so >> gpurun_out/abr2.jsonl 2>> gpurun_out/abr2.err
  VB_WORK=$W VB_OPTS=14=$O VB_TAG=":occ$O" python scripts/variant_bench.py build/variants/lib_o_noeset.so >> gpurun_out/abr2.jsonl 2>> gpurun_out/abr2.err
done
VB_WORK=$W VB_OPTS=14=2 VB_TAG=":occ2b" python scripts/variant_bench.py build/variants/lib_a_base.so >> gpurun_out/abr2.jsonl 2>> gpurun_out/abr2.err
echo done
