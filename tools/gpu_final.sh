#!/bin/bash
# Round-2 evidence session: GPU tests + bench + launch list + ncu captures (tools/gpu_round.sh), then the
# other configs' bench lines (tools/gpu_configs.sh).
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
rm -rf gpurun_out/parity
bash tools/gpu_round.sh r2
TAG=r2 bash tools/gpu_configs.sh
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r2/smoke.log
