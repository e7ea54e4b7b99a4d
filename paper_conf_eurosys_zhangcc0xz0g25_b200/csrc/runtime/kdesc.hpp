// kdesc.hpp -- launch descriptor of one tenant kernel (host side).
//
// Built once per kernel at bl_append_kernel (validation, tile count, grid,
// TMA tensor maps) so that a launch on the hot path is a single
// cudaLaunchKernel with a precomputed parameter block plus the per-launch
// gate arguments (SM range, slot, sequence number).
#pragma once
#include <cuda_runtime_api.h>

#include <cstdint>
#include <string>

#include "../../../include/bless/bless.h"
#include "../kernels/executor.cuh"

namespace bless {

struct KernelDesc;
typedef cudaError_t (*LaunchFn)(const KernelDesc&, const GateArgs&, cudaStream_t);

struct KernelDesc {
  bl_op op{};
  const char* family = "";
  uint32_t tiles = 1;
  int grid = 0, block = 0, smem = 0;
  int max_occ = 8;         // blocks-per-SM cap of the grid (measured per family, profiles/round1/occ_cap.txt)
  int grid_full = 0;       // uncapped full-occupancy grid: used whenever the launch range is restricted
  int S = 0;               // SMs of the device (a launch over [0, S) may use the capped grid)
  double flops = 0;        // algorithmic FLOPs per launch (roofline)
  double bytes = 0;        // algorithmic HBM bytes per launch (roofline)
  LaunchFn launch = nullptr;
  const void* kernel_fn = nullptr;  // for the occupancy query (grid = S x blocks/SM)
  void* owned = nullptr;   // device scratch owned by this kernel (split-K workspace), cudaFree'd with it
  int choice_bn = 0, choice_splits = 0, choice_bk = 0, choice_halo = 0, choice_mt = 0;  // tcgen05 tile config (0 = not tc)
  bool counts_done = false;  // can count finished units / wait on a predecessor's count (GateArgs dep_*)
  alignas(128) unsigned char params[4096];  // family-specific parameter block
};

// Grid of one launch: the capped grid only for an unrestricted range -- a
// restricted launch needs the full-occupancy grid so that lingering
// out-of-range CTAs can never absorb it (gate_linger in executor.cuh).
inline int launch_grid(const KernelDesc& d, const GateArgs& g) {
  return (d.grid_full > 0 && g.hi - g.lo < d.S) ? d.grid_full : d.grid;
}

struct DeviceCaps {
  int S = 148;             // SMs
  int cc_major = 10, cc_minor = 0;
  int smem_optin = 232448;
};

// Validate op and fill the descriptor.  Returns false with err on a bad op.
bool build_kernel(const bl_op& op, const DeviceCaps& caps, KernelDesc& out, std::string& err);

// Per-family builders (return true if they took the op).
bool build_simt(const bl_op& op, const DeviceCaps& caps, KernelDesc& out, std::string& err);
// tcgen05 GEMM/conv: tile configuration (BN, split-K factor); zero = the
// builder's default heuristic.  tc_candidates lists the configurations the
// registration-time autotuner times for one op (returns how many).
struct TcChoice {
  int bn = 0, splits = 0;
  int bk = 0;   // K depth per pipeline stage (64 or 128; 0 = the builder's default)
  int halo = 0; // 1: halo implicit-GEMM conv (one input box per channel chunk serves all 3x3 taps)
  int mt = 0;   // M tile rows: 256 = two M = 128 MMAs per K step (GEMM / 1x1), 0/128 = one
};
bool build_tc_gemm(const bl_op& op, const DeviceCaps& caps, KernelDesc& out, std::string& err,
                   const TcChoice* force = nullptr);
int tc_candidates(const bl_op& op, const DeviceCaps& caps, TcChoice* out, int max);
bool build_gemv_tma(const bl_op& op, const DeviceCaps& caps, KernelDesc& out, std::string& err);
bool build_nn(const bl_op& op, const DeviceCaps& caps, KernelDesc& out, std::string& err);
bool build_attn_tc(const bl_op& op, const DeviceCaps& caps, KernelDesc& out, std::string& err);

}  // namespace bless
