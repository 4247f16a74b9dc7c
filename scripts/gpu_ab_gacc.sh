# A/B: Alley's compensated sums in global memory (GSWORD_SMEM_ACC=2) vs shared memory
set -u
mkdir -p gpurun_out
VB_WORK=${VB_WORK:-C1:1,C1:2,C1:0,C2:0} python scripts/variant_bench.py build/variants/lib_u_head.so build/variants/lib_v_gacc.so > gpurun_out/abg.jsonl 2> gpurun_out/abg.err
echo done
