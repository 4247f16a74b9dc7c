#!/bin/bash
# Final validation call: build, GPU suite, smoke, the bench line (plain and under torchrun with
# one rank, the driver's launch form) and the reference arm.  usage: bash scripts/gpu_call_final.sh r02o
set -u
cd "$(dirname "$0")/.."
TAG=${1:-final}
mkdir -p gpurun_out
make all > gpurun_out/${TAG}_build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/${TAG}_pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1
echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
timeout 900 python bench.py > gpurun_out/${TAG}_bench.jsonl 2> gpurun_out/${TAG}_bench.err
timeout 600 python bench.py --impl reference > gpurun_out/${TAG}_bench_reference.jsonl 2> gpurun_out/${TAG}_bench_reference.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29517 \
    bench.py --gpus 1 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_torchrun.jsonl 2> gpurun_out/${TAG}_bench_torchrun.err
echo done
