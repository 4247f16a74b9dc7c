# Autotune consistency: each library twice (fresh processes, so fresh autotunes)
set -u
mkdir -p gpurun_out
W=${VB_WORK:-C1:1,C1:2,C1:0,C2:0,C3:0}
for rep in 1 2; do
VB_WORK=$W VB_TAG=":r$rep" python scripts/variant_bench.py build/variants/lib_a_base.so build/variants/lib_p_tune.so build/variants/lib_q_tune8.so >> gpurun_out/abt2.jsonl 2>> gpurun_out/abt2.err
done
echo done
