// kernels.cuh -- launcher interfaces between the C-ABI layer (api.cu) and the kernel files.
#pragma once
#include <vector>

#include "common.cuh"

namespace fp {

constexpr int kSplitMaxCS = 8;

// What a CSR plan precomputes for the column-split cluster kernel (csr_colsplit.cuh); soff is
// device memory owned by the plan (fp_csr_plan).
struct CsrSplit {
  const int32_t* soff = nullptr;  // [(cs-1)][m]: entries of row r with column < cb[k+1]
  int cs = 0;                     // CTAs per cluster = column blocks
  int cb[kSplitMaxCS + 1] = {};   // column block bounds, cb[0] = 0, cb[cs] = n
  int width = 0;                  // max_k cb[k+1] - cb[k]
};

struct PatternArgs {
  int64_t m = 0, n = 0;
  // dense
  const void* X = nullptr;
  int64_t ld = 0;
  // csr
  int64_t nnz = 0;
  const int64_t* rowptr = nullptr;
  const int32_t* colidx = nullptr;
  const void* val = nullptr;
  // vectors / scalars
  const void* y = nullptr;
  const void* v = nullptr;
  const void* z = nullptr;
  double alpha = 1.0, beta = 0.0;
  void* w = nullptr;
  fp_dtype dtype = FP_F64;
  // when false the CTA-finalise does NOT add beta*z (multi-GPU ranks != 0); set by dist layer
  bool add_beta_z = true;
  // when true the result is ADDED to the current w (w += alpha X^T(v (.) X y) [+ beta z]);
  // used by the host-streaming (out-of-core) path to sum row chunks
  bool accumulate = false;
  // row epilogue (aggregate.cuh fpd::RowEpi): 0 = Eq. (1) (optionally writing X y to row_out),
  // 1 = logistic-regression gradient (v = labels, writes D to row_out, loss to scalar_out)
  int epi_kind = 0;
  double epi_c = 1.0;
  void* row_out = nullptr;
  double* scalar_out = nullptr;
  // column split of a CSR plan (FP_VAR_CSR_COLSPLIT only)
  const CsrSplit* split = nullptr;
};

// Dense chooser (B200 plan): fills vs, tl, bs, grid, variant ... for the kernels in dense.cu.
fp_status plan_dense(const PatternArgs& a, int device, fp_launch* out);
fp_status launch_dense(const PatternArgs& a, const fp_launch& L, cudaStream_t s);

fp_status plan_csr(const PatternArgs& a, int device, fp_launch* out);
fp_status launch_csr(const PatternArgs& a, const fp_launch& L, cudaStream_t s);
// Column-split cluster plan for a CSR matrix whose y / w blocks fit shared memory: fills
// L (variant FP_VAR_CSR_COLSPLIT) and the host part of sp (cs, cb, width); cs_force = 0 picks
// the smallest cluster that fits.  Returns false if no cluster size fits.
bool plan_colsplit(const PatternArgs& a, int device, int cs_force, CsrSplit* sp, fp_launch* L);

// api.cu: validation + alpha == 0 path + plan + launch of one pattern evaluation
fp_status run_csr(const PatternArgs& a, const fp_launch* override_, cudaStream_t s);
PatternArgs csr_args(int64_t m, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx,
                     const void* val, const void* y, const void* v, const void* z, double alpha, double beta, void* w,
                     fp_dtype dtype);

// Variant 17 (csr_binned.cu): binned producer + fixed-point consumer + exact finalize.
fp_status launch_binned(const PatternArgs& a, const fp_launch& L, int64_t y_prefix, cudaStream_t s);
int binned_nbin(int64_t n);     // 1 or 2 column blocks; 0 if n is too wide
int binned_producer_regs(bool has_y);
// Variant 18 (csr_binned.cu): flat-4 kernel with the fixed-point CTA partial (small n).
fp_status launch_flat4_fixed(const PatternArgs& a, const fp_launch& L, cudaStream_t s);
size_t flat4_fixed_smem(int64_t n, fp_dtype dt, bool has_y);
int flat4_fixed_blocks_per_sm(int64_t n, fp_dtype dt, bool has_y);

// Variant 19 (csr_packed.cu): a column-blocked copy of a CSR matrix (fp_csr_plan_pack) and
// Eq. (1) on it with one CTA group per column split (y + fixed-point w in shared memory).
constexpr int kPkMaxCS = 8;
struct Packed {
  int64_t m = 0, n = 0, nnz = 0;
  int cs = 0, bw = 0, groups = 0;
  int64_t ntiles = 0, entries = 0, max_tiles_per_warp = 0;
  const int64_t* rowptr = nullptr;
  uint4* tile_desc = nullptr;           // [cs][ntiles] (offset / 4, length, first row, rows)
  int32_t* wtile = nullptr;             // [groups * 32 + 1]
  uint32_t* cr = nullptr;               // [entries] column in block | row in tile << 16
  void* val = nullptr;                  // [entries] fp32 / fp64
  fp_dtype dtype = FP_F32;
  int bs = 1024;                        // threads per CTA of the pass
  int ns1 = 0;                          // cs == 1: tile slots per warp of k_pk1's shared-memory ring
  unsigned long long* xch = nullptr;    // exchange slots
  unsigned* epoch = nullptr;            // call counter
  double* part = nullptr;               // [groups][n]
  double* spill = nullptr;              // [cs][bw + 1]
  unsigned long long* trace = nullptr;  // FP_PK_TRACE measurement buffer
  int trace_warps = 32;                 // warps per CTA of the pass (trace layout)
  // mode 1 = variant 20 (csr_l2block.cu): cs L2-sized column blocks of bw columns, chunks
  // (tile_desc) of block b = [l2cb[b], l2cb[b + 1]); the heaviest block is processed last (fused)
  int mode = 0;
  int heavy = 0;
  std::vector<int64_t> l2cb;
  double* rowdot = nullptr;             // [m]: row dots p, then q
  int cbits = 0;                        // column bits of the entry word
  int nhot = 0;                         // hot columns: hcol[slot], entries hrow / hval by column,
  int32_t* hcol = nullptr;              //   work items hitems (first entry, count, slot)
  uint32_t* hrow = nullptr;
  void* hval = nullptr;
  uint4* hitems = nullptr;
  int64_t nhitems = 0;
  int64_t hot_entries = 0;
  uint32_t* dotlist = nullptr;          // variant 20: the dot phase's chunks in (row panel, block) order
  int64_t ndot = 0;
  int64_t heavy_entries = 0;            // stored entries of the fused block
};
// variant 20 (csr_l2block.cu)
int64_t l2block_bw(int64_t n, fp_dtype dt);
fp_status l2block_build(int64_t m, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx,
                        const void* val, fp_dtype dtype, Packed* p, cudaStream_t s);
fp_status l2block_exec(Packed* p, const PatternArgs& a, cudaStream_t s);
void l2block_launch(const Packed* p, fp_launch* L);
void packed_detail(const Packed* p, int64_t out[8]);  // fp_csr_plan_pack_detail
int packed_cs(int64_t n, fp_dtype dt);  // column blocks (1, 2, 4, 8) for n columns, 0 if too wide
fp_status packed_build(int64_t m, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx,
                       const void* val, fp_dtype dtype, int cs_force, Packed** out, cudaStream_t s);
fp_status packed_exec(Packed* p, const PatternArgs& a, cudaStream_t s);
}  // namespace fp
struct fp_csr_plan;
namespace fp {
// csr_plan.cu: one evaluation on a plan's matrix (packed copy when a.val == NULL)
fp_status plan_run(const fp_csr_plan* p, PatternArgs& a, cudaStream_t s);
void plan_shape(const fp_csr_plan* p, int64_t* m, int64_t* n, int64_t* nnz, const int64_t** rowptr,
                const int32_t** colidx, fp_dtype* dt);
void packed_free(Packed* p);
void packed_launch(const Packed* p, fp_launch* L);

size_t binned_ws_bytes(int64_t n, int64_t nnz, int nbin, int producer_grid, int consumers);

// w = beta*z (or 0): the alpha == 0 / m == 0 path, and the pre-initialisation of the L2 path.
fp_status launch_scale_z(int64_t n, const void* z, double beta, void* w, fp_dtype dt, cudaStream_t s);

// Register count of the kernel instantiation a plan selects (0 if unknown).
int dense_kernel_regs(const PatternArgs& a, const fp_launch& L);

}  // namespace fp
