# GPU suite on the default build, then A/B of the previous build against it (autotuned)
set -u
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/abt_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/abt_pytest.log
W=${VB_WORK:-C1:1,C1:2,C1:0,C2:0,C3:0,C3:1,C0:0}
VB_WORK=$W python scripts/variant_bench.py build/variants/lib_a_base.so build/variants/lib_p_tune.so > gpurun_out/abt.jsonl 2> gpurun_out/abt.err
echo done
