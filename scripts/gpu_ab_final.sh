# GPU suite + A/B (previous build vs the default build) + bench line
set -u
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/abf_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/abf_pytest.log
W=${VB_WORK:-C1:1,C1:2,C1:0,C2:0,C3:0,C3:1}
VB_WORK=$W python scripts/variant_bench.py build/variants/lib_a_base.so build/variants/lib_r_final.so > gpurun_out/abf.jsonl 2> gpurun_out/abf.err
timeout 900 python bench.py > gpurun_out/abf_bench.jsonl 2> gpurun_out/abf_bench.err
echo done
