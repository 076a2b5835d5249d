#!/bin/bash
# A/B timing of build/libve_*.so variants only (no tests)
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
bash scripts/ab.sh
