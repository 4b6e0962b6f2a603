// internal.h — geometry shared by the host API (polyconv.cu) and the kernels.
// Product code only; nothing here is used by oracle/.
#pragma once
#include <cstdint>
#include <cstddef>
#include <cuda_runtime.h>

namespace polyconv {

// Operand storage formats produced by packing (reading R11).
enum Fmt : int { FMT_F32 = 0, FMT_TF32 = 1, FMT_BF16 = 2 };

// Problem geometry, all derived once in polyconv_plan.
struct Geom {
  int N, C, H, W, K, R, S, sh, sw, ph, pw;
  int P, Q;             // output size
  int Hp, Wp;           // padded input size; Wp is the row pitch Iw of Eq. 10
  long long L_A;        // Hp*Wp, input polynomial length (Eq. 10)
  long long L_U;        // (R-1)*Wp + S, kernel polynomial length (P.1378-1380)
  long long M_ext;      // positions per image that can hold an output:
                        // (P-1)*sh*Wp + (Q-1)*sw + 1 (last extraction degree - (L_U-1) + 1)
  int Cp, Kp;           // padded channel counts of the interleaved layouts
  int urep;             // copies of the tap-major filter in the plan workspace (>= 1): the
                        // tensor-core MAC spreads its filter reads over them (every CTA
                        // streams the whole filter; one copy is an L2 hot spot)
};

inline int fmt_bytes(int f) { return f == FMT_BF16 ? 2 : 4; }

// ---- pack.cu ------------------------------------------------------------
cudaError_t launch_pack_input_planar(const Geom& g, const void* x, bool x_bf16, void* dst,
                                     int fmt, cudaStream_t st);
cudaError_t launch_pack_input_interleaved(const Geom& g, const void* x, bool x_bf16, void* dst,
                                          int fmt, cudaStream_t st);
cudaError_t launch_pack_filter_planar(const Geom& g, const void* w, bool w_bf16, void* dst,
                                      int fmt, cudaStream_t st);
cudaError_t launch_pack_filter_tapmajor(const Geom& g, const void* w, bool w_bf16, void* dst,
                                        int fmt, int Kp, int Cp, cudaStream_t st);
// stride-2 phase-split filter [R'*S'][Kp][Cp] (bf16 in / out, mac_hankel phase mode, reading R19)
cudaError_t launch_pack_filter_phase(const Geom& g, const void* w, void* dst, int Rp, int Sp, int php, int pwp,
                                     int Kp, int Cp, cudaStream_t st);
// fused: input interleaved + filter tap-major in one launch
cudaError_t launch_pack_both_interleaved(const Geom& g, const void* x, const void* w, bool io_bf16,
                                         void* xdst, void* wdst, int fmt, cudaStream_t st);

// ---- mac_1x1.cu (1x1 stride-1 unpadded, BF16: x read as the MN-major operand) ----
bool mac1x1_supported(const Geom& g, int fmt, bool io_bf16);
// 0: x is read in place; else the pitch of the gathered position operand [N*C][pitch]
int mac1x1_pitch(const Geom& g);
cudaError_t launch_gather1x1(const Geom& g, const void* x, void* xq, cudaStream_t st);
// x: NCHW input (pitch 0) or the gathered copy; U: tap-major packed filter [1][Kp][Cp],
// Kp % 128 == 0, Cp % 64 == 0; launched as a programmatic dependent of the filter pack
cudaError_t launch_mac_1x1(const Geom& g, const void* x, const void* U, int Kp, int Cp, void* y, int num_sms,
                           cudaStream_t st, char* err, size_t errlen);

// ---- polyphase.cu (stride s: phases of the padded input as channels, reading R4b) ----
// xq [N][s*s*C][Hq][Wq] and wq [K][s*s*C][Rq][Sq] in the io dtype
cudaError_t launch_polyphase(const Geom& g, int Hq, int Wq, int Rq, int Sq, const void* x, const void* w, void* xq,
                             void* wq, bool io_bf16, cudaStream_t st);

// ---- extract.cu -----------------------------------------------------------
cudaError_t launch_extract(const Geom& g, const float* coeffs, void* y, bool y_bf16,
                           cudaStream_t st);

// ---- mac_thin.cu ----------------------------------------------------------
// A: planar packed input [N][C][L_A] (fmt); U: tap-major packed filter [RS][Kp][Cp] (fmt)
cudaError_t launch_mac_thin(const Geom& g, const void* A, const void* U, int Kp, int Cp, int fmt,
                            void* y, bool y_bf16, cudaStream_t st);

// ---- mac_fp32.cu ----------------------------------------------------------
struct Fp32Tiling { int cc; int smem_bytes; int smax; };
Fp32Tiling fp32_tiling(const Geom& g);
// x: NCHW input (f32 or bf16); U: tap-major fp32 filter [RS][Kp][Cp]; y: NCHW output (x's dtype)
cudaError_t launch_mac_fp32(const Geom& g, const Fp32Tiling& t, const void* x, bool io_bf16, const float* U,
                            int Kp, int Cp, void* y, cudaStream_t st);
inline int fp32_kp(int K) { return (K + 63) / 64 * 64; }

// ---- mac_tc.cu ------------------------------------------------------------
struct TcTiling {
  int bm;          // positions per tile (UMMA M) = 128
  int bn;          // output channels per tile (UMMA N), multiple of 32, <= 256
  int kc;          // channels per k-block (row of the smem operand)
  int row_bytes;   // kc * element bytes: 32, 64 or 128 (= swizzle width)
  int stages;      // smem pipeline depth
  int smem_bytes;  // dynamic shared memory
  int tmem_cols;   // TMEM allocation (2 accumulators)
  int num_m, num_n, kblocks;
  int grid;        // persistent CTAs
};
bool tc_supported(const Geom& g, int fmt);
TcTiling tc_tiling(const Geom& g, int fmt, int num_sms);
// A: interleaved packed input [N*L_A][Cp]; U: tap-major packed filter [RS][Kp][Cp]
cudaError_t launch_mac_tc(const Geom& g, const TcTiling& t, int fmt, const void* A, const void* U,
                          void* y, bool y_bf16, cudaStream_t st, char* err, size_t errlen);

// ---- mac_tc2.cu (default tensor-core path: window reuse across taps) ----------
struct Tc2Tiling {
  int nt;          // positions per tile (UMMA N), multiple of 16, <= 256
  int kc;          // channels per chunk (one swizzle row)
  int row_bytes;   // kc * element bytes: 32, 64 or 128
  int nr;          // kernel rows served by one position window
  int ngroups;     // ceil(R / nr)
  int brows;       // rows of one position window (multiple of 32)
  int num_mt, num_kt, num_tiles, nchunks;
  int cs;          // cluster size (CTAs sharing multicast filter tiles)
  int num_groups;  // cluster work items: ceil(num_mt / cs) * num_kt
  int a_stages;    // filter ring depth (stages)
  int tps;         // filter taps per stage
  int mode;        // 0: windows by TMA from the packed input; 1/2: fused packers (TMA staging / loads)
  bool tma_x;      // fused: raw input staged by TMA (x as [N*C][H*W], 16-byte row pitch) vs direct loads
  int box_bytes, stg_bytes;
  int smem_bytes, acc_stride, tmem_cols, grid;
  int ecols, stage_pitch, stage_bytes;  // epilogue staging
};
bool tc2_supported(const Geom& g, int fmt);
// true when a fused tiling packs the input with the ring-staged 8x8-transpose packers
bool tc2_is_mx(const Tc2Tiling& t);
Tc2Tiling tc2_tiling(const Geom& g, int fmt, bool x_bf16, int num_sms, bool fused, bool y_bf16);
// mode 0: A = interleaved packed input [N*L_A][Cp] (x unused); fused modes:
// x = NCHW input (packed on the fly), A unused.  U: tap-major packed filter
// [RS][Kp][Cp], Kp % 128 == 0.  pdl: launch as a programmatic dependent of the
// preceding pack kernel, which it waits for before reading A / U.
// fused modes with w != nullptr: the kernel packs the filter itself (a3) into U,
// every CTA one slice, synchronised through *fcount (must reach ftarget =
// number of launches so far x t.grid; the plan owns the counter).
cudaError_t launch_mac_tc2(const Geom& g, const Tc2Tiling& t, int fmt, const void* x, bool x_bf16,
                           const void* A, const void* U, void* y, bool y_bf16, bool pdl, cudaStream_t st,
                           char* err, size_t errlen, const void* w = nullptr,
                           unsigned long long* fcount = nullptr, unsigned long long ftarget = 0);

// ---- mac_pair.cu (bf16 default: one launch, CTA pairs, resident filter) -------
struct PairTiling {
  bool ok;              // shape supported (bf16 math, K <= 256, filter half + 2 windows fit)
  int kc, row_bytes;    // channels per chunk (one swizzle row of kc bf16 words)
  int Cp, NN;           // padded channels (multiple of kc); MMA N = padded output channels
  int nchunks, RS, nblk;
  int box_rows, nbox;   // position window: nbox TMA boxes of box_rows rows
  int wbytes, wbytes_tx, fbytes;
  int ring;             // window ring depth
  int smem_bytes, tmem_cols;
  int num_tiles, num_pairs, grid;
  int rb, nb, nunits, spitch;  // packing bands (rb padded rows, nb per image), staging pitch
  int pack_tma;                // bands in/out by TMA (x band box ne_box x C; A boxes 64 ch x rb*Wp rows)
  int ne_box, last_rows, in_bytes, obox_bytes, obox_bytes2;
  int tr, tpi, ntile;          // row-aligned CTA tiles: tr output rows of one image each
  int epi_tma, estage_bytes;   // epilogue staged in shared memory and written by TMA stores
  int u_img0;  // first image whose bands the pack writes (0)
  int split, pack_grid, pack_smem;    // packing in its own grid, the pair kernel its programmatic dependent
};
PairTiling pair_tiling(const Geom& g, int fmt, bool io_bf16, int num_sms);
// One launch: packs w -> U [R*S][NN][Cp] and x -> A [N*L_A][Cp] (bf16, plan workspace),
// meets on *fcount (must reach ftarget = launches so far x t.grid), then the pair MAC.
// fcount: filter-slice counter (ftarget = launches so far x t.grid); bflag: [N*t.nb] band
// flags (zeroed once; band u is published as `epoch` = launches so far); state: launch
// cache from pair_state_new() (tensor maps + parameters per pointer set), or nullptr
cudaError_t launch_mac_pair(const Geom& g, const PairTiling& t, const void* x, const void* w, bool io_bf16,
                            void* A, void* U, void* y, cudaStream_t st, char* err, size_t errlen, void* state);
void* pair_state_new();
void pair_state_free(void* s);

// ---- mac_hankel.cu (persistent CTA-pair kernel fed from NCHW x; reading R16 layout) ----
struct HankelTiling {
  bool ok;
  int pitch, HS, delta;    // input polynomial row pitch, image stride (rows), origin shift
  int PT;                  // 256-position units
  int Cp, nchunks;         // channels padded to whole 128-byte operand rows
  int NN, NB, Kp;          // MMA N (output channels per block), blocks, padded K of U
  int T;                   // 128-position tiles per CTA per item (accumulators share filter blocks)
  int wrows, wslots;       // window rows per slot, window ring depth
  int fslots, resident;    // filter blocks in shared memory; 1 = whole filter half resident
  int aligned;             // every position pair is one aligned input pair (fast loader)
  uint32_t wslot_bytes, fblk_bytes;
  int smem_bytes, tmem_cols, npairs, grid;
  int nacc;  // TMEM accumulator buffers (1 or 2)
  // stride-2 phase mode (reading R19): the kernel runs on the phase-split geometry
  int phase, eC, eH, eW, eR, eS, eph, epw;
  int kc;  // channels per window row: 64 bf16 / 32 tf32 (128 B), 16 bf16 (32 B, small-C phase mode)
  // plane-staged loader: whole (image, 64-channel) blocks of x by bulk copy, two staging buffers
  int planes, pimg_max;
  uint32_t pimg_bytes;
  int rowtile;  // the stem: pitch 128, one output row per tile, TMA-stored epilogue
};
HankelTiling hankel_tiling(const Geom& g, int fmt, int num_sms, bool io_bf16);
// x: NCHW input (io dtype); U: tap-major packed filter [RS][Kp][Cp] (t.Kp, t.Cp), packed by
// the preceding launch, which this one follows as a programmatic dependent
// zero: device buffer of hankel_zero_bytes(g) zero bytes (read in place of padding)
size_t hankel_zero_bytes(const Geom& g);
// ys[0..nys-1]: outputs [N][ktot][P][Q]; this plan's K channels go to channel offset koff of each
cudaError_t launch_mac_hankel(const Geom& g, const HankelTiling& t, int fmt, const void* x, bool io_bf16,
                              const void* U, void* const* ys, int nys, int ktot, int koff, const void* zero,
                              cudaStream_t st, char* err, size_t errlen);

// ---- fft.cu (R = IFFT(FFT(A) . FFT(U)) per channel, summed in frequency) ----
struct FftTiling {
  bool ok;
  int L, logL, F;          // FFT length (power of two >= L_A + L_U - 1), bins kept (L/2 + 1)
  int RB;                  // (n, k) rows per CTA of the inverse transform
  size_t x_bytes, u_bytes, y_bytes, tw_bytes;  // spectra X^[F][N][C], U^[F][K][C], Y^[F][N][K]; twiddles
};
FftTiling fft_tiling(const Geom& g);
cudaError_t launch_fft_twiddles(const FftTiling& t, void* tw, cudaStream_t st);
// ws: x_bytes + u_bytes + y_bytes; tw: twiddles from launch_fft_twiddles
cudaError_t launch_fft_conv(const Geom& g, const FftTiling& t, const void* x, const void* w, bool io_bf16, void* ws,
                            const void* tw, void* y, cudaStream_t st);

}  // namespace polyconv
