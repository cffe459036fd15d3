// Kernel launch parameters of the transfer engine (host <-> device contract).
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include "engine.cuh"

namespace adapcc {

constexpr int kMaxRanksDev = 64;

struct LaunchParams {
  const Task* tasks;
  const BufRef* refs;
  const FlagRef* flags;
  const Item* items;
  uint32_t nitems;
  int dtype;
  int nranks;
  int my_rank;        // multi-process: this rank; loopback: -1
  int ipc;            // 1: multi-process start check + done post
  int drop_rank;      // test hook (loopback): tasks owned by this rank are skipped
  uint64_t epoch;     // flag value of this launch (monotonic per communicator)
  uint64_t timeout_ns;
  unsigned* counters; // device: [0] work cursor, [1] finished CTAs, [2] abort
  int* err;           // host-mapped error word
  char* send[kMaxRanksDev];
  char* recv[kMaxRanksDev];
  char* arena[kMaxRanksDev];  // parity half of each rank's arena (peer-mapped)
  char* hdr[kMaxRanksDev];    // arena header of each rank (done epoch at +0)
};

int engine_threads();
cudaError_t engine_occupancy(int dtype, int* blocks_per_sm);
cudaError_t engine_launch(const LaunchParams& p, int grid, cudaStream_t stream);

}  // namespace adapcc
