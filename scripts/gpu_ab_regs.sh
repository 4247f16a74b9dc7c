# A/B of the register-pressure changes: previous build; new build autotuned, forced occupancy 0 and 2
set -u
mkdir -p gpurun_out
W=${VB_WORK:-C1:1,C1:2,C1:0,C2:0,C3:0}
VB_WORK=$W python scripts/variant_bench.py build/variants/lib_a_base.so > gpurun_out/abr.jsonl 2> gpurun_out/abr.err
for O in -1 0 2; do
  VB_WORK=$W VB_OPTS=14=$O VB_TAG=":occ$O" python scripts/variant_bench.py build/variants/lib_n_regs.so >> gpurun_out/abr.jsonl 2>> gpurun_out/abr.err
done
echo done
