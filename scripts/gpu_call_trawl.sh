# trawling A/B call: parity tests of both enumeration kernels, then scripts/trawl_eval.py on C2
set -u
make all > gpurun_out/tw_build.log 2>&1 || { tail gpurun_out/tw_build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "${TW_TESTS:-trawl or large_query}" > gpurun_out/tw_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/tw_pytest.log
timeout 900 python scripts/trawl_eval.py --config C2 > gpurun_out/tw_c2.jsonl 2> gpurun_out/tw_c2.err
echo done
