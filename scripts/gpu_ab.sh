# A/B call: GPU tests on the default build, then variant_bench over build/variants/*.so
set -u
make all > gpurun_out/ab_build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q ${AB_TESTS:-} > gpurun_out/ab_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/ab_pytest.log
VB_WORK=${VB_WORK:-C1:1,C1:0,C2:0,C3:0} timeout 1200 python scripts/variant_bench.py ${AB_LIBS:-build/variants/*.so} > gpurun_out/ab_variants.jsonl 2> gpurun_out/ab_variants.err
echo done
