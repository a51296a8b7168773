#!/bin/bash
# compute-sanitizer over reduced GPU parity cases (run on the GPU box through gpurun, from the repo root):
#   tools/sanitize.sh <round>
# memcheck (out-of-bounds / misaligned / leaks of device memory), racecheck and synccheck (shared
# memory hazards, barrier misuse) on the hot kernels (k_fwd_fast / k_fwd_fix, k_rev_fast / k_rev_fix, k_map_pd,
# k_unmap_sh, k_slots with and without shadows), the queued re-map / release (leases), the glue interpreter, the peer-copy path and the smoke test.
set -u
R=${1:-r02}
mkdir -p gpurun_out/$R
CASES="tests/test_gpu_parity.py::test_scalar_map_unmap_release tests/test_gpu_parity.py::test_mapArray_roundtrip_permutation tests/test_gpu_parity.py::test_random_device_slices[shadow-8] tests/test_gpu_deferred.py::test_deferred_released_by_matching_unmap[shadow] tests/test_gpu_deferred.py::test_deferred_slots_rewritten_by_gpu[shadow] tests/test_gpu_glue.py tests/test_gpu_group.py::test_handoff_through_a_dirty_peer tests/test_gpu_leases.py::test_leased_releases_match_the_oracle[shadow]"
for tool in memcheck racecheck synccheck; do
  extra=""
  [ "$tool" = memcheck ] && extra="--leak-check full"
  PYTORCH_NO_CUDA_MEMORY_CACHING=1 timeout 2400 compute-sanitizer --tool $tool $extra --error-exitcode 17 --target-processes all \
    python -m pytest $CASES -q -x -p no:cacheprovider > gpurun_out/$R/sanitize_$tool.log 2>&1
  echo "rc=$?" >> gpurun_out/$R/sanitize_$tool.log
  tail -5 gpurun_out/$R/sanitize_$tool.log
done
timeout 600 compute-sanitizer --tool memcheck --error-exitcode 17 python -c "import __graft_entry__ as g; g.smoke()" \
  > gpurun_out/$R/sanitize_smoke.log 2>&1
echo "rc=$?" >> gpurun_out/$R/sanitize_smoke.log
tail -3 gpurun_out/$R/sanitize_smoke.log
