#!/bin/bash
# Final round-2 validation of the last build: GPU suite, smoke, sanitizers, launch list + ncu of the
# bench kernels (profile_round.sh), bench line (plain and torchrun N = 1) and reference arm.
# usage (on the GPU box): bash scripts/gpu_call_r02s.sh r02s
set -u
cd "$(dirname "$0")/.."
TAG=${1:-r02s}
mkdir -p gpurun_out profiles
make all > gpurun_out/${TAG}_build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/${TAG}_pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1
echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
for T in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $T --error-exitcode 9 python scripts/sanitize.py > gpurun_out/${TAG}_san_$T.log 2>&1
  echo "$T rc=$?" >> gpurun_out/${TAG}_sanitizers.txt
  tail -3 gpurun_out/${TAG}_san_$T.log >> gpurun_out/${TAG}_sanitizers.txt
done
bash scripts/profile_round.sh ${TAG} > gpurun_out/${TAG}_profile_round.log 2>&1
cp profiles/traffic_latest.json gpurun_out/${TAG}_traffic_latest.json
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29519 \
    bench.py --gpus 1 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_torchrun.jsonl 2> gpurun_out/${TAG}_bench_torchrun.err
echo done
