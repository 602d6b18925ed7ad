// kernels.h — launch interface between the host runtime (api.cpp) and the
// sm_100a device kernels (life.cu, conv.cu).  Internal to libmapsm.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace mapsm {

// How a kernel maps an input row index y outside [0, rows) of its slab
// (see mapsm_halo_kind in include/mapsm.h).
enum RowMap : int {
    ROWMAP_HALO = 0,   // read the slab buffer's halo row (exchanged, or zeroed for ZERO)
    ROWMAP_WRAP = 1,   // g == 1 WRAP: y mod rows (no halo copy needed)
    ROWMAP_CLAMP = 2   // global edge under CLAMP: nearest owned edge row
};

// Column boundary == the grid's boundary (columns are never split).
enum ColMode : int { COL_WRAP = 0, COL_CLAMP = 1, COL_ZERO = 2 };

// What a launcher actually launched (mapsm_launch_query): the kernel, its
// grid, and for the row-streaming ring kernels the band table the CTAs split
// (tma_rows.cuh seg_iter), so the host can report rows per CTA segment.
enum LaunchKernel : int {
    LK_NONE = 0, LK_LIFE_TMA = 1, LK_LIFE_REG = 2, LK_LIFE_ANYW = 3, LK_LIFE_PERSIST = 4, LK_LIFE_TB = 5,
    LK_CONV_TMA = 6, LK_CONV_REG = 7, LK_CONV_GENERIC = 8, LK_CONV_WIDE = 9, LK_CONV3D = 10,
    LK_LIFE_TB_PERSIST = 11, LK_CONV_TB2 = 12
};
struct LaunchRec {
    int kernel = LK_NONE;
    int64_t ctas = 0;
    int threads = 0, smem = 0;
    int ring_stages = 0;     // NS of the shared-memory ring (0: no ring)
    int rows_per_stage = 0;  // input rows per ring stage
    int consumer_warps = 0;
    int64_t nstrips = 0;     // column strips of a row
    int nbands = 0;
    int64_t begin[3] = {0, 0, 0}, end[3] = {0, 0, 0};
    int64_t cta_begin[4] = {0, 0, 0, 0};
    int gens = 1;            // generations per launch
};

// One stencil launch over a slab.  `in`/`out` point at owned row 0 of the
// input/output slab buffers; halo rows live at rows -r..-1 and rows..rows+r-1.
struct StencilGeom {
    const void* in;
    void* out;
    int64_t pitch;   // bytes between rows (same for in and out)
    int64_t rows;    // owned rows of the slab
    int64_t w;       // columns (cells)
    int top_map, bot_map, col_mode;
    // Window(3D) grids: `rows` counts planes, `pitch` is the plane pitch, and a
    // plane holds plane_rows rows of rpitch bytes (0 for 2-D grids)
    int64_t plane_rows = 0, rpitch = 0;
    LaunchRec* rec = nullptr;  // filled by the launcher when non-null
    int wslot = -1;            // conv r >= 3: the grid's weight slot (conv_upload_weights)
    bool pdl = true;           // programmatic dependent launch on the previous kernel of the stream
                               // (off in the concurrent-boundary schedules: an early-scheduled
                               // interior grid would take the SMs kept for the boundary launch)
};

// fp32 conv, r = 2..4 (FFMA2 kernels): weights live in __constant__ slots,
// uploaded once per grid and device (conv_upload_weights, at bind); at most
// kConvWeightSlots such grids at a time.  No-op for other radii.
constexpr int kConvWeightSlots = 32;
constexpr int kConvMaxPairs = 72, kConvMaxTaps = 81;
cudaError_t conv_upload_weights(int r, int col_mode, int slot, const float* weights);
bool conv_uses_weight_slot(int r);  // the radii whose kernels read a weight slot (FFMA2 pairs)

// Output-row bands computed by one launch (1 band = all rows or interior;
// 2 bands = the boundary rows [0,r) and [rows-r,rows)).
struct RowBands {
    int64_t begin[3], end[3];
    int nbands;
};

// Fused peer-memory halo exchange of one launch (see tma_rows.cuh); all-null
// = plain launch.  Pointers may address a peer GPU's memory (CUDA IPC).
struct FusedLink {
    void* mailbox;          // this slab's tma::Mailbox
    void* dst_up;           // up neighbour: out-parity buffer at its bottom-halo row 0
    void* dst_down;         // down neighbour: out-parity buffer at its top-halo row -r
    unsigned int* sig_up;   // up neighbour's mailbox.recv_bot
    unsigned int* sig_down; // down neighbour's mailbox.recv_top
    int wait_top, wait_bot;
    int ce = 0;             // copy-engine exchange: the halos arrive by peer memcpy; the mailbox
                            // counters hold the sender's generation count (wait until >= mine)
};

// Life (bit-packed: bit j of 32-bit word m of a row = column 32m + j).
// `resident_warps` = warps the device keeps resident for this kernel
// (persistent-style row chunking); 0 = compute from the occupancy API.
cudaError_t launch_life_step(const StencilGeom& g, const RowBands& b, int num_sms, cudaStream_t s,
                             const FusedLink* link = nullptr);
// n generations of a whole slab (no exchanged halos) in ONE cooperative
// launch with a grid barrier between generations; g.in/g.out are the buffers
// of generation 0 / 1 (generation n ends in g.in if n is even, else g.out).
// `bar` = one device word of barrier state.
cudaError_t launch_life_persistent(const StencilGeom& g, int64_t n, unsigned int* bar, int num_sms, cudaStream_t s);
// n generations of a whole slab (no exchanged halos) resident in SHARED
// memory (life_resident.cu): one cooperative launch of `ctas` CTAs (one per
// SM), K generations between neighbour-only halo exchanges through `xbuf`
// (life_resident_xbuf_bytes) with `flags` (ctas words).  Generation n is
// written to g.out (always, whatever the parity of n).  life_resident_plan:
// false if the slab does not fit (w % 128, shared-memory capacity).
bool life_resident_plan(int64_t w, int64_t rows, int num_sms, int* ctas, int* K, int* smem);
int64_t life_resident_xbuf_bytes(int64_t w, int ctas, int K);
cudaError_t launch_life_resident(const StencilGeom& g, int64_t n, int ctas, int K, int smem, uint32_t* xbuf,
                                 unsigned int* flags, cudaStream_t s);
// K generations of Life in ONE temporally blocked launch (life_tb.cu): reads
// input rows [-K, rows+K) of g.in (halo rows must be valid to depth K; under
// ROWMAP_CLAMP the rows outside are the MIRROR image), writes owned rows of
// the bands of generation t+K to g.out.  zero_top / zero_bot: ZERO global
// edges (rows outside the slab forced to 0 at every generation).
bool life_tb_supported(int k);
cudaError_t launch_life_tb(const StencilGeom& g, const RowBands& b, int k, int zero_top, int zero_bot, int num_sms,
                           cudaStream_t s);
cudaError_t launch_pack_life(const uint8_t* src, int64_t src_pitch, void* dst, int64_t dst_pitch,
                             int64_t rows, int64_t w, cudaStream_t s);
cudaError_t launch_unpack_life(const void* src, int64_t src_pitch, uint8_t* dst, int64_t dst_pitch,
                               int64_t rows, int64_t w, cudaStream_t s);

// fp32 window convolution, radius r in 1..8, weights (2r+1)^2 row-major
// (r <= 4: TMA row pipeline, conv_impl.cuh; r = 5..8: shared-memory tiles,
// conv_wide.cu).
cudaError_t launch_conv_step(const StencilGeom& g, const RowBands& b, int r, const float* weights,
                             int num_sms, cudaStream_t s, const FusedLink* link = nullptr);
// Two generations of the fp32 convolution in ONE pass (conv_tb.cuh), r = 1..2,
// w % 4 == 0: reads g.in rows [-2r, rows+2r) (halo rows valid to depth 2r,
// i.e. MAPSM_OPT_DEEP_HALO = 2), writes generation t+2 of the bands to g.out.
bool conv_tb2_supported(int r, int64_t w, int64_t pitch);
cudaError_t launch_conv_tb2(const StencilGeom& g, const RowBands& b, int r, int zero_top, int zero_bot, int num_sms,
                            cudaStream_t s);

// Window(3D) fp32 convolution (conv3d.cu), radius 1..2, (2r+1)^3 weights
// ordered (dz, dy, dx); bands are plane ranges; col_mode is the y/x boundary.
cudaError_t launch_conv3d(const StencilGeom& g, const RowBands& b, int r, const float* weights, int num_sms,
                          cudaStream_t s);

cudaError_t launch_conv_wide(const StencilGeom& g, const RowBands& b, int r, const float* weights, cudaStream_t s);

// Reductive (Static) output: 256-bin histogram of a u8 slab into out[256]
// (zeroed here; 64-bit counts); and the sum of g partial histograms.
cudaError_t launch_histogram(const uint8_t* img, int64_t pitch, int64_t w, int64_t rows, unsigned long long* out,
                             int num_sms, cudaStream_t s);
// Single-launch variant (one slab, one process): CTAs commit into `acc`
// (256 counts + a CTA ticket at acc[256], all zero on entry and left zero on
// exit); the last CTA to commit moves the counts to final_out[256] and
// re-zeroes acc.  No memset, no copy.
cudaError_t launch_histogram_final(const uint8_t* img, int64_t pitch, int64_t w, int64_t rows,
                                   unsigned long long* acc, unsigned long long* final_out, int num_sms,
                                   cudaStream_t s);
// Chained histogram tasks over stencil grids (api.cpp mapsm_task_histogram):
// Life (bit-packed rows; bins 0 = dead, 1 = alive) and fp32 (bin =
// floor(v * 256) clamped).  `out` is zeroed here.
cudaError_t launch_histogram_life(const void* bits, int64_t pitch, int64_t w, int64_t rows, unsigned long long* out,
                                  int num_sms, cudaStream_t s);
cudaError_t launch_histogram_f32(const float* img, int64_t pitch, int64_t w, int64_t rows, unsigned long long* out,
                                 int num_sms, cudaStream_t s);
cudaError_t launch_histogram_sum(const unsigned long long* const* parts_dev, int g, unsigned long long* out,
                                 cudaStream_t s);

}  // namespace mapsm
