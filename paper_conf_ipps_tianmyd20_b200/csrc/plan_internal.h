// Internal plan layout shared by the host planner (planner.cpp) and the
// device side (pcgcn_api.cu).  Not part of the ABI.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "../../include/pcgcn.h"

namespace pcgcn {

constexpr int TILE_M = 128;  // dense row tile: destination rows (UMMA M)
constexpr int TILE_K = 32;   // dense chunk: source columns (one 128-byte tf32 K-major row)

struct DevicePlan {
  bool built = false;
  float* r = nullptr;             // [n] plan order
  int64_t* sp_rowptr = nullptr;   // [rows+1] shard-local, rebased to 0
  int32_t* sp_col = nullptr;      // [nnz_s shard]
  int32_t* zd_index = nullptr;    // [rows] shard-local row tile slot (t*128+rr), -1 none
  int32_t* rt_row0 = nullptr;     // [nrt shard] plan row
  int32_t* rt_nrows = nullptr;    // [nrt shard]
  int64_t* rt_cptr = nullptr;     // [nrt+1] rebased
  int32_t* rt_order = nullptr;    // [nrt] full-mode engine tile order (balanced, see upload_plan)
  int32_t* rt_bysize = nullptr;   // [nrt] tiles by descending chunk count (dynamic largest-first claims)
  int32_t* ch_col0 = nullptr;     // [nch shard]
  uint32_t* bits = nullptr;       // [nch*128]
  float* zd = nullptr;            // [nrt*128*fpad_max] dense partial sums
  float* yhi = nullptr;           // [2*fpad_max x n_pad] tf32 split of the (prescaled) input, feature-major:
                                  // rows [0,npad) hi, rows [npad,2npad) lo for a call of width npad
  float* ypre = nullptr;          // [n*fpad_max] prescaled copy for un-prescaled inputs
  float* zrow = nullptr;          // [256] zeros
  int32_t* row_seg = nullptr;     // [rows] first long-row segment, -1 none (nullptr if nseg == 0)
  int64_t* seg_lo = nullptr;      // [nseg] shard-local edge range of each segment
  int64_t* seg_hi = nullptr;
  float* seg_ws = nullptr;        // [nseg x fpad_max] segment partial sums
  int32_t* seg_row = nullptr;     // [nseg] shard-local row of each segment
  int32_t* seg_cnt = nullptr;     // [nseg] inline-segment completion counts (zero between calls)
  int* counter = nullptr;         // [32] selective-pass row ticket
  int32_t* halo_send = nullptr;   // [Σ_q send rows] plan rows of this shard, peers in rank order
  int32_t* halo_recv = nullptr;   // [Σ_q recv rows] plan rows of other shards, peers in rank order
  int64_t halo_nsend = 0, halo_nrecv = 0;
  int64_t rows = 0, nnz_s = 0, nrt = 0, nch = 0, nseg = 0;
  int64_t n_pad = 0;
  int fpad_max = 0;
  int64_t bytes = 0;
  std::vector<void*> owned;
  void* ev[5] = {nullptr, nullptr, nullptr, nullptr, nullptr};  // PCGCN_PROFILE events (cudaEvent_t)
  bool ev_used[4] = {false, false, false, false};
  void* side = nullptr;                    // cudaStream_t: segment pass overlapped with the full mode
  void* ev_fork = nullptr;                 // cudaEvent_t (timing disabled)
  void* ev_join = nullptr;
};

}  // namespace pcgcn

struct pcgcn_plan_s {
  int64_t n = 0;
  int64_t nnz_t = 0;  // nnz(Ã)
  int32_t P = 0;
  float theta = 0.f;
  pcgcn_opts opts{};
  int32_t sweeps = 0;
  int64_t clusters = 0;
  std::vector<int32_t> part, perm;
  std::vector<int64_t> pstart;
  std::vector<float> r;
  std::vector<int32_t> blk_k, blk_i;
  std::vector<int64_t> blk_nnz;
  std::vector<uint8_t> blk_dense;
  std::vector<int64_t> sp_rowptr;
  std::vector<int32_t> sp_col;
  std::vector<int32_t> rt_row0, rt_nrows;
  std::vector<int64_t> rt_cptr;
  std::vector<int32_t> ch_col0;
  std::vector<uint32_t> bits;
  std::vector<int32_t> zd_index;
  // shard
  int32_t k_lo = 0, k_hi = 0;
  int64_t row_lo = 0, row_hi = 0, rt_lo = 0, rt_hi = 0;
  std::vector<int64_t> shard_row0;                 // [world+1] first plan row of every shard
  std::vector<std::vector<int32_t>> halo_recv;     // [world] rows of shard q this shard reads
  std::vector<std::vector<int32_t>> halo_send;     // [world] rows of this shard that shard q reads
  int64_t stats_src_rows_pc = 0, stats_shard_src_rows_pc = 0;
  pcgcn_stats stats{};
  pcgcn::DevicePlan d;
};

namespace pcgcn {
// host planner (planner.cpp); fills every host array and stats (not device)
pcgcn_status build_host_plan(const pcgcn_csr* A, int32_t P, float theta, const pcgcn_opts* o,
                             pcgcn_plan_s* p);
// device side (pcgcn_api.cu)
pcgcn_status upload_plan(pcgcn_plan_s* p);
void free_device_plan(pcgcn_plan_s* p);
void set_error(const std::string& msg);
}  // namespace pcgcn
