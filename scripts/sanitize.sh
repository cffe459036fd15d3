#!/usr/bin/env bash
# compute-sanitizer over the engine kernels (run on the GPU box via gpurun):
#   memcheck  - out-of-bounds / misaligned global + shared accesses, leaks
#   racecheck - shared-memory hazards (item header, TMA smem ring)
#   synccheck - illegal __syncthreads / barrier use
#   initcheck - reads of uninitialised device memory (arenas, flag regions)
# Each tool runs a loopback GPU-test subset covering both kernels and both
# plan kinds; logs go to gpurun_out/sanitize_<tool>.log.
set -u
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
CS="compute-sanitizer --target-processes all --print-limit 20 --error-exitcode 9"
run() {
  local tool=$1 files=$2 sel=$3 extra=${4:-}
  echo "== $tool: $files -k '$sel' $extra" > gpurun_out/sanitize_$tool.log
  ADAPCC_TIMEOUT_MS=120000 timeout 1500 $CS --tool $tool $extra \
    python -m pytest $files -q -p no:cacheprovider -k "$sel" \
    >> gpurun_out/sanitize_$tool.log 2>&1
  echo "== exit $?" >> gpurun_out/sanitize_$tool.log
}
LB=tests/test_gpu_loopback.py
MORE="tests/test_gpu_primitives.py tests/test_gpu_late_join.py tests/test_gpu_a2a_routes.py tests/test_gpu_trace.py"
# r02 paths: STAGED late join (both kernels), bulk reduce-add ACCUMULATE, NVLS on the emulated switch,
# link probes, the online coordinator (loopback)
R02="tests/test_gpu_nvls.py tests/test_gpu_link_probe.py tests/test_gpu_coordinator.py"
# leak-check off: the only leaks reported are PyTorch caching-allocator segments alive at exit
run memcheck "$LB $MORE $R02" "not watchdog and not multiprocess and not racing and not loopback_profile and not messages_scale"
run racecheck "$LB" "(allreduce_parity and f32 and (stars8 or dbinary)) or (alltoall and bf16) or c1_config or (tma_large_items and f32)"
run synccheck "$LB tests/test_gpu_late_join.py tests/test_gpu_nvls.py" "(allreduce_parity and (stars8 or ring)) or allgather or c1_config or (deterministic and staged) or emulated or subnormal"
run initcheck "$LB tests/test_gpu_late_join.py" "(allreduce_parity and f32 and stars8) or c1_config or (alltoall and i32) or (deterministic and staged and f32)"
# racecheck's model of mbarrier handoffs (the TMA kernel's item queue): a
# textbook correct producer/consumer handoff via mbarriers (A) vs named barriers (B)
nvcc -gencode arch=compute_100a,code=sm_100a -o gpurun_out/rc_probe scripts/debug/racecheck_mbarrier_probe.cu \
  && for v in A B; do
       echo "== racecheck probe $v" >> gpurun_out/sanitize_racecheck_probe.log
       compute-sanitizer --tool racecheck --print-limit 4 gpurun_out/rc_probe $v >> gpurun_out/sanitize_racecheck_probe.log 2>&1
       echo "== exit $?" >> gpurun_out/sanitize_racecheck_probe.log
     done
rm -f gpurun_out/rc_probe
