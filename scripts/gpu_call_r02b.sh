#!/bin/bash
# GPU call: full GPU suite (kernel changes), smoke, candidate-graph layout report.
set -u
cd "$(dirname "$0")/.."
TAG=${1:-r02b}
mkdir -p gpurun_out
make all > gpurun_out/${TAG}_build.log 2>&1
timeout 2700 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/${TAG}_pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1
echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
timeout 1800 python scripts/cg_layout_report.py > gpurun_out/${TAG}_cg_layout.jsonl 2> gpurun_out/${TAG}_cg_layout.err
echo "cg rc=$?" >> gpurun_out/${TAG}_cg_layout.err
echo done
