# Autotune decisions, disjoint steady-state pilots: 3 fresh processes per library
set -u
mkdir -p gpurun_out
W=${VB_WORK:-C1:2,C1:1,C3:0}
for rep in 1 2 3; do
VB_WORK=$W VB_SAMPLES=1e8 VB_TAG=":r$rep" python scripts/variant_bench.py build/variants/lib_t_disj4.so >> gpurun_out/abt3.jsonl 2>> gpurun_out/abt3.err
done
echo done
