set -u
make all > gpurun_out/s3_build.log 2>&1 || exit 1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "large_query or trawl" > gpurun_out/s3_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/s3_pytest.log
: > gpurun_out/r02k_sanitizers.txt
for T in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $T --error-exitcode 9 python scripts/sanitize.py > gpurun_out/r02k_san_$T.log 2>&1
  echo "$T rc=$?" >> gpurun_out/r02k_sanitizers.txt
  tail -3 gpurun_out/r02k_san_$T.log >> gpurun_out/r02k_sanitizers.txt
done
