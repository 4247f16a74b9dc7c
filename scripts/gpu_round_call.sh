set -u
make all > gpurun_out/r01c_build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r01c_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r01c_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r01c_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r01c_smoke.log
bash scripts/profile_round.sh r01c
