// The C ABI of libstarsim.so (include/starsim.h): handle lifecycle, argument validation, scratch arena,
// stream-ordered orchestration of the sm_100a kernels, per-kernel CUDA-event timing, error strings.
#include <cmath>
#include <cstdio>
#include <algorithm>
#include <cstring>
#include <string>
#include <vector>

#include "../../include/starsim.h"
#include "common.cuh"
#include "launch.h"
#include "plan.cuh"

using namespace starsim;

namespace {

thread_local std::string g_create_error;

struct Buf {
  void* p = nullptr;
  size_t cap = 0;
};

struct Launch {
  int kclass;
  int n;  // kernels enqueued between the two events
  cudaEvent_t a, b;
};

}  // namespace

// A captured render (CUDA graph) and the arguments it was captured with: replayed when a call repeats them.
struct GraphKey {
  const void *x, *y, *mag, *out;
  const uint32_t* n_dev;
  int64_t n;
  int32_t W, H, row0, rows, R, obits, psf, tile_impl, bin_impl, ndst;
  float* dst[MAX_DST];
  float sigma, gain;
  cudaStream_t st;
  uint64_t scratch_gen;
  bool operator==(const GraphKey& o) const {
    return x == o.x && y == o.y && mag == o.mag && out == o.out && n_dev == o.n_dev && n == o.n && W == o.W && H == o.H &&
           row0 == o.row0 && rows == o.rows && R == o.R && obits == o.obits && psf == o.psf && tile_impl == o.tile_impl && bin_impl == o.bin_impl && ndst == o.ndst &&
           std::equal(dst, dst + MAX_DST, o.dst) && sigma == o.sigma && gain == o.gain && st == o.st &&
           scratch_gen == o.scratch_gen;
  }
};

struct starsim_ctx {
  int dev = 0;
  int num_sms = 148;
  int32_t psf = 0;  // starsim_set_psf: 0 point-sampled Eq. 2, 1 pixel-integrated (NEXT-2)
  int32_t roi = 0;  // starsim_set_roi: 0 square, 1 pixel circle (NEXT-3; atomic and lookup-table renders only)
  int32_t tile_impl = 0;  // starsim_set_tile_kernel: 0 auto, 1 lists, 2 sorted bins, 3 warp-specialised sorted bins
  int32_t bin_impl = 0;   // starsim_set_binning: 0 auto (dbin.cu when it applies), 1 always bin.cu's pipeline
  std::string err;
  const uint32_t* n_dev = nullptr;  // starsim_set_star_count: device-resident star count of the tiled renders
  int dfused_grid = 0;              // largest co-resident k_dfused grid (0: the three-kernel binning only)
  bool ws_presort = false;          // k_tile_ws reads chunks presorted by k_chsort (env STARSIM_WS_PRESORT=1; slower)
  Buf rec, slots, ids, tmp, tile_off, items, split_tab, parts, partial, zeroed, stage, cmat, codes, segs, srec, sbin, sext,
      rblk, cbin, gbar;
  uint64_t scratch_gen = 0;  // bumped whenever a scratch buffer moves (invalidates the captured graph)
  // last tiled render, for starsim_get_bins
  bool have_bins = false;
  cudaStream_t last_stream = nullptr;
  int64_t last_ntiles = 0;
  // the last tiled render took the sparse path (no CSR built): starsim_get_bins bins these arrays on demand
  bool last_sparse = false;
  struct {
    const float *x, *y, *m;
    int64_t n;
    FrameParams fp;
    int tps, part_cap;
  } sp{};
  // CUDA graph of the last render signature (non-default streams only; STARSIM_NO_GRAPH=1 disables)
  bool use_graphs = true;
  bool have_graph = false;
  GraphKey gkey{};
  cudaGraphExec_t gexec = nullptr;
  // profiling
  bool prof = false;
  std::vector<cudaEvent_t> ev_pool;
  std::vector<Launch> pending;
  double ms[STARSIM_NUM_KCLASS] = {};
  int64_t launches[STARSIM_NUM_KCLASS] = {};
};

namespace {

struct DevGuard {
  int prev = -1;
  explicit DevGuard(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DevGuard() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

int fail(starsim_ctx* c, int code, const std::string& msg) {
  if (c) c->err = msg;
  return code;
}

int cuda_fail(starsim_ctx* c, cudaError_t e, const char* where) {
  return fail(c, e == cudaErrorMemoryAllocation ? STARSIM_ENOMEM : STARSIM_ECUDA,
              std::string(where) + ": " + cudaGetErrorString(e));
}

// Grow a scratch buffer geometrically (x1.5); contents are not preserved.
int grow(starsim_ctx* c, Buf& b, size_t bytes, const char* what) {
  if (bytes <= b.cap) return STARSIM_OK;
  size_t want = b.cap + b.cap / 2;
  if (want < bytes) want = bytes;
  if (want < 4096) want = 4096;
  c->scratch_gen++;
  if (b.p) {
    cudaFree(b.p);  // implicitly synchronises the device: earlier calls that used b are done
    b.p = nullptr;
    b.cap = 0;
  }
  cudaError_t e = cudaMalloc(&b.p, want);
  if (e != cudaSuccess) {
    cudaGetLastError();
    e = cudaMalloc(&b.p, bytes);  // retry without headroom
    if (e != cudaSuccess) {
      cudaGetLastError();
      b.p = nullptr;
      return fail(c, STARSIM_ENOMEM, std::string("cudaMalloc(") + what + ", " + std::to_string(bytes) + " B) failed");
    }
    want = bytes;
  }
  b.cap = want;
  return STARSIM_OK;
}

cudaEvent_t get_event(starsim_ctx* c) {
  if (!c->ev_pool.empty()) {
    cudaEvent_t e = c->ev_pool.back();
    c->ev_pool.pop_back();
    return e;
  }
  cudaEvent_t e = nullptr;
  cudaEventCreate(&e);
  return e;
}

// Run `launch` on stream st, bracketed by CUDA events on the same stream when profiling is on.
template <typename F>
void timed(starsim_ctx* c, int kclass, cudaStream_t st, F&& launch, int nlaunch = 1) {
  if (!c->prof) {
    launch();
    return;
  }
  Launch l{kclass, nlaunch, get_event(c), get_event(c)};
  cudaEventRecord(l.a, st);
  launch();
  cudaEventRecord(l.b, st);
  c->pending.push_back(l);
}

int check_launch(starsim_ctx* c, const char* where) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(c, e, where);
  return STARSIM_OK;
}

int validate_frame(starsim_ctx* c, const float* x, const float* y, const float* mag, int64_t n, int32_t W, int32_t H,
                   float sigma, int32_t R, float gain, const void* out) {
  if (n < 0) return fail(c, STARSIM_EINVAL, "n < 0");
  if (n > 0 && (!x || !y || !mag)) return fail(c, STARSIM_EINVAL, "n > 0 with a NULL x, y or mag");
  if (n > 0xFFFFFFFFll) return fail(c, STARSIM_EINVAL, "n >= 2^32 (star indices are 32-bit)");
  if (!out) return fail(c, STARSIM_EINVAL, "out is NULL");
  if (W < 1 || W > STARSIM_MAX_DIM || H < 1 || H > STARSIM_MAX_DIM)
    return fail(c, STARSIM_EINVAL, "width/height outside [1, 32767]");
  if ((int64_t)W * H >= (1ll << 31)) return fail(c, STARSIM_EINVAL, "width*height >= 2^31");
  if (!std::isfinite(sigma) || !(sigma > 0.f)) return fail(c, STARSIM_EINVAL, "sigma not finite or <= 0");
  if (R < 1 || R > STARSIM_MAX_ROI) return fail(c, STARSIM_EINVAL, "roi outside [1, 255]");
  if (!std::isfinite(gain) || gain < 0.f) return fail(c, STARSIM_EINVAL, "gain not finite or < 0");
  return STARSIM_OK;
}

FrameParams make_params(int32_t W, int32_t H, int32_t row0, int32_t rows, float sigma, int32_t R, float gain,
                        int32_t psf) {
  FrameParams fp;
  fp.W = W;
  fp.H = H;
  fp.row0 = row0;
  fp.rows = rows;
  fp.R = R;
  fp.ntx = (W + TILE_W - 1) / TILE_W;
  fp.nty = (rows + TILE_H - 1) / TILE_H;
  const double s = (double)sigma;
  fp.sk = (float)std::sqrt(1.0 / (2.0 * s * s * std::log(2.0)));  // exp(-d^2/(2 s^2)) = 2^(-(d sk)^2)
  fp.s_scale = (double)gain / (2.0 * M_PI * s * s);          // Eq. 1 gain with Eq. 2's 1/(2 pi s^2)
  fp.psf = psf;
  fp.roi = 0;
  fp.tile_impl = 0;
  fp.bin_impl = 0;
  fp.ndst = 0;
  for (int i = 0; i < MAX_DST; ++i) fp.dst[i] = nullptr;
  fp.n_dev = nullptr;
  fp.lite = 0;
  fp.obits = 0;
  fp.vec = 0;
  fp.vec32 = 0;
  fp.kint = (float)(1.0 / (std::sqrt(2.0) * s));
  // the part / segment length of long tile lists (reading R19): shorter for the wide-ROI kernel, whose stars cost
  // R^2 FMAs each (a heavy tile then spreads over more CTAs)
  fp.split = wide_ok(R) ? WIDE_SPLIT : SPLIT_LEN;
  if (psf) fp.s_scale = (double)gain;  // the pixel masses of the integrated PSF are already normalised
  return fp;
}

// the deterministic binning of dbin.cu applies (DB_MAXT tiles, an ROI over at most 2 x 2 tiles)
bool dbin_ok(const FrameParams& fp, int64_t ntiles) { return fp.bin_impl == 0 && ntiles <= DB_MAXT && fp.R <= DB_MAXR; }

int tiles_per_axis(int R, int tile, int ntiles_axis) {
  int t = (R - 1 + tile - 1) / tile + 1;
  return t < ntiles_axis ? t : ntiles_axis;
}

// k_tile_ws with its chunks presorted by k_chsort (STARSIM_WS_PRESORT=1 at context creation; measured slower at T:
// k_chsort 21 us against 6 us saved in k_tile_ws)
bool ws_presort(const starsim_ctx* c, const FrameParams& fp) {
  return c->ws_presort && fp.tile_impl == STARSIM_TILE_WS && fp.R <= SB_MAXR;
}

// Enqueue the tiled render on stream st: memset of the header + tile counters, k_prep, k_scan, k_scatter,
// k_sortlists, k_tile.
int enqueue_binning(starsim_ctx* c, const float* x, const float* y, const float* mag, int64_t n,
                    const FrameParams& fp, int64_t ntiles, int tps, int part_cap, cudaStream_t st) {
  Header* hdr = (Header*)c->zeroed.p;
  uint32_t* cnt = (uint32_t*)(hdr + 1);
  const size_t zbytes = sizeof(Header) + sizeof(uint32_t) * (CNT_STRIDE + 1) * (size_t)ntiles;
  uint32_t* done = cnt + CNT_STRIDE * ntiles;
  uint32_t* ids = (uint32_t*)c->ids.p;
  uint32_t* tile_off = (uint32_t*)c->tile_off.p;
  uint32_t* slots = (uint32_t*)c->slots.p;
  StarRec* rec = (StarRec*)c->rec.p;
  const int plan = plan_word(part_cap, fp.split);  // the planner's pool size and part length (plan.cuh)
  int rc;
  if (dbin_ok(fp, ntiles)) {
    // deterministic counting sort (dbin.cu): no memset, no atomics on global counters, no per-tile sort
    // (step a2 runs inside k_dplace; an empty catalogue has no k_dplace, so k_scan plans its all-empty tiles)
    uint32_t* C = (uint32_t*)c->cmat.p;
    if (n > 0 && dsmall_ok(n)) {
      // at most DB_CTA stars: the whole binning in one CTA, one launch (k_dsmall)
      timed(c, 0, st, [&] {
        launch_dsmall(x, y, mag, n, fp, rec, (int)ntiles, tile_off, hdr, (WorkItem*)c->items.p,
                      (uint2*)c->split_tab.p, plan, done, ids, st);
      });
      if ((rc = check_launch(c, "k_dsmall"))) return rc;
    } else if (n > 0 && c->dfused_grid > 0 && dfused_block_ok(n) && dbin_ctas(n) <= c->dfused_grid) {
      // every CTA of the catalogue resident: count, column scan and placement in one cooperative launch (k_dfused)
      cudaError_t le = cudaSuccess;
      timed(c, 0, st, [&] {
        le = launch_dfused(x, y, mag, n, fp, rec, C, cnt, (int)ntiles, tile_off, hdr, (WorkItem*)c->items.p,
                           (uint2*)c->split_tab.p, plan, done, ids, (uint32_t*)c->gbar.p, st);
      });
      if (le != cudaSuccess) return cuda_fail(c, le, "k_dfused (cooperative launch)");
      if ((rc = check_launch(c, "k_dfused"))) return rc;
    } else if (n > 0) {
      timed(c, 0, st, [&] { launch_dcount(x, y, mag, n, fp, rec, (uint32_t*)c->codes.p, C, (int)ntiles, st); });
      if ((rc = check_launch(c, "k_dcount"))) return rc;
      timed(c, 2, st, [&] { launch_dcolscan(C, n, (int)ntiles, cnt, 1, fp.n_dev, st); });  // dense totals for k_dplace
      if ((rc = check_launch(c, "k_dcolscan"))) return rc;
      timed(c, 1, st, [&] {
        launch_dplace((const uint32_t*)c->codes.p, n, fp, C, (int)ntiles, cnt, tile_off, hdr, (WorkItem*)c->items.p,
                      (uint2*)c->split_tab.p, plan, done, ids, st);
      });
      if ((rc = check_launch(c, "k_dplace"))) return rc;
    } else {
      timed(
          c, 2, st,
          [&] {
            launch_dcolscan(C, n, (int)ntiles, cnt, CNT_STRIDE, nullptr, st);
            launch_scan(cnt, ntiles, tile_off, hdr, (WorkItem*)c->items.p, (uint2*)c->split_tab.p, plan,
                        c->partial.p, done, st);
          },
          1 + scan_launches(ntiles));
      if ((rc = check_launch(c, "k_dcolscan/k_scan"))) return rc;
    }
  } else {
    timed(c, 5, st, [&] { cudaMemsetAsync(hdr, 0, zbytes, st); });
    if (n > 0) {
      timed(c, 0, st, [&] { launch_prep(x, y, mag, n, fp, rec, cnt, slots, tps, st); });
      if ((rc = check_launch(c, "k_prep"))) return rc;
    }
    timed(
        c, 2, st,
        [&] {
          launch_scan(cnt, ntiles, tile_off, hdr, (WorkItem*)c->items.p, (uint2*)c->split_tab.p, plan,
                      c->partial.p, done, st);
          launch_scatter(rec, n, fp, slots, tps, tile_off, ids, st);
        },
        (n > 0 ? 1 : 0) + scan_launches(ntiles));
    if ((rc = check_launch(c, "k_scan/k_scatter"))) return rc;
    timed(c, 1, st, [&] { launch_sortlists(ids, (uint32_t*)c->tmp.p, tile_off, ntiles, n, st); });
    if ((rc = check_launch(c, "k_sortlists"))) return rc;
  }
  return STARSIM_OK;
}

int enqueue_tiled(starsim_ctx* c, const float* x, const float* y, const float* mag, int64_t n, const FrameParams& fp,
                  int64_t ntiles, int tps, int part_cap, void* out, cudaStream_t st, bool sparse) {
  int rc;
  if (sparse) {
    // the sparse path (tile_sb.cu): records, then one CTA per tile that builds its own list -- no binning launches
    timed(c, 0, st, [&] { launch_srec(x, y, mag, n, fp, (StarRec*)c->rec.p, (uint32_t*)c->codes.p, st); });
    if ((rc = check_launch(c, "k_srec"))) return rc;
    timed(c, 3, st, [&] {
      launch_tile_sparse((const StarRec*)c->rec.p, (const uint32_t*)c->codes.p, n, fp, out, (float*)c->segs.p, st);
    });
    return check_launch(c, "k_tile_sparse");
  }
  if ((rc = enqueue_binning(c, x, y, mag, n, fp, ntiles, tps, part_cap, st))) return rc;
  Header* hdr = (Header*)c->zeroed.p;
  uint32_t* cnt = (uint32_t*)(hdr + 1);
  uint32_t* done = cnt + CNT_STRIDE * ntiles;
  uint32_t* ids = (uint32_t*)c->ids.p;
  uint32_t* tile_off = (uint32_t*)c->tile_off.p;
  StarRec* rec = (StarRec*)c->rec.p;
  (void)cnt;
  if (fp.tile_impl == STARSIM_TILE_T8 && fp.R <= SB_MAXR) {
    // k_t8sort: every tile list segment sorted by ROI corner bin, records written in that order (tile8.cu)
    timed(c, 1, st, [&] {
      launch_t8sort(ids, rec, fp, (WorkItem*)c->items.p, part_cap, hdr, (StarRec*)c->srec.p, (uint32_t*)c->sbin.p,
                    (uint32_t*)c->sext.p, st);
    });
    if ((rc = check_launch(c, "k_t8sort"))) return rc;
    timed(c, 3, st, [&] {
      launch_tile8((StarRec*)c->srec.p, fp, out, (WorkItem*)c->items.p, (uint2*)c->split_tab.p, (float*)c->parts.p,
                   part_cap, done, (float*)c->segs.p, hdr, (const uint32_t*)c->sbin.p, (const uint32_t*)c->sext.p,
                   c->num_sms, st);
    });
  } else {
    const bool pre = ws_presort(c, fp);
    if (pre) {
      // k_chsort: k_tile_ws's per-chunk corner-bin sort done ahead (records in walk order, bin starts per chunk)
      timed(c, 1, st, [&] {
        launch_chsort(ids, rec, fp, (WorkItem*)c->items.p, part_cap, hdr, (StarRec*)c->srec.p, (uint16_t*)c->cbin.p,
                      st);
      });
      if ((rc = check_launch(c, "k_chsort"))) return rc;
    }
    timed(
        c, 3, st,
        [&] {
          launch_tile(ids, rec, fp, out, (WorkItem*)c->items.p, (uint2*)c->split_tab.p, (float*)c->parts.p, part_cap,
                      done, hdr, c->num_sms, st, (float*)c->segs.p, tile_off, pre ? (StarRec*)c->srec.p : nullptr,
                      pre ? (uint16_t*)c->cbin.p : nullptr);
        },
        fp.lite ? 2 : 1);
  }
  if ((rc = check_launch(c, "k_tile"))) return rc;
  return STARSIM_OK;
}

int render_tiled(starsim_ctx* c, const float* x, const float* y, const float* mag, int64_t n, int32_t W, int32_t H,
                 int32_t row0, int32_t rows, float sigma, int32_t R, float gain, int32_t obits, void* out,
                 cudaStream_t st, float* const* dsts = nullptr, int ndst = 0) {
  DevGuard g(c->dev);
  FrameParams fp = make_params(W, H, row0, rows, sigma, R, gain, c->psf);
  fp.obits = obits;
  fp.tile_impl = c->tile_impl;
  fp.roi = c->roi;
  // NEXT-3: the circle mask lives in k_tile_sb's walk (R <= SB_MAXR) and in k_tile's (wider ROIs)
  if (fp.roi) fp.tile_impl = STARSIM_TILE_SB;
  if (fp.tile_impl == STARSIM_TILE_AUTO) {
    // the warp-specialised kernel wins on dense frames (its per-item pipeline latency and static item order cost
    // more than they save on sparse, clustered and integrated-PSF frames: DESIGN.md §9): expected list length per
    // tile for a uniform field, n (128 + R - 1)(64 + R - 1) / (W rows).  k_tile8 (STARSIM_TILE_T8) is faster in the
    // tile kernel but needs the k_t8sort pass: a slower frame at T, so it is opt-in.
    const double per_tile = (double)n * (TILE_W + R - 1) * (TILE_H + R - 1) / ((double)W * (rows > 0 ? rows : 1));
    // (wide ROIs: STARSIM_TILE_SB = k_tile_wide, measured faster than its warp-specialised form k_tile_wws)
    fp.tile_impl = (c->psf == 0 && per_tile >= WS_MIN_PER_TILE && !wide_ok(R)) ? STARSIM_TILE_WS : STARSIM_TILE_SB;
  }
  fp.bin_impl = c->bin_impl;
  fp.n_dev = c->n_dev;
  // k_tile_sb hands the light tiles to k_tile_lite (same bits; tile_sb.cu)
  // (worth its second launch on frames of many mostly-light tiles: measured, DESIGN.md §9 -- C3 with 1K / 16K
  // stars gains 4-6 us; C1, C2 and fig2, with few tiles or ~50 stars per tile, lose 2-8 us)
  {
    const double per_tile = (double)n * (TILE_W + R - 1) * (TILE_H + R - 1) / ((double)W * (rows > 0 ? rows : 1));
    const int64_t nt = (int64_t)fp.ntx * fp.nty;
    fp.lite = (fp.tile_impl == STARSIM_TILE_SB && R <= SB_MAXR && LITE_MAX > 0 && per_tile <= LITE_AUTO_PER_TILE &&
               nt >= LITE_AUTO_TILES) ? 1 : 0;
  }
  // the sparse path (AUTO, <= SPARSE_MAX stars): no binning launches, the same image bit for bit (tile_sb.cu)
  const bool sparse = c->tile_impl == STARSIM_TILE_AUTO && c->bin_impl == STARSIM_BIN_AUTO &&
                      fp.tile_impl == STARSIM_TILE_SB && R <= SB_MAXR &&
                      sparse_ok(n, (int64_t)fp.ntx * fp.nty);
  // one vector store per 8-pixel run: 32 B (fp32) / 8 B (u8) / 16 B (u16); rows must keep that alignment
  const int vb = obits == 8 ? 8 : 16;
  bool aligned = ((uintptr_t)out % vb) == 0;
  fp.ndst = ndst;
  for (int i = 0; i < ndst; ++i) {
    fp.dst[i] = dsts[i] + (int64_t)row0 * W;  // band origin inside destination frame i
    aligned = aligned && ((uintptr_t)fp.dst[i] % vb) == 0;
  }
  fp.vec = ((W * (obits ? obits / 8 : 4)) % vb == 0 && aligned) ? 1 : 0;
  bool al32 = ((uintptr_t)out % 32) == 0;
  for (int i = 0; i < ndst; ++i) al32 = al32 && ((uintptr_t)fp.dst[i] % 32) == 0;
  fp.vec32 = (obits == 0 && (W * 4) % 32 == 0 && al32) ? 1 : 0;
  const int64_t ntiles = (int64_t)fp.ntx * fp.nty;
  const int tps = tiles_per_axis(R, TILE_W, fp.ntx) * tiles_per_axis(R, TILE_H, fp.nty);
  const int64_t pmax = n * (int64_t)tps;
  if (pmax >= 0xFFFFFFFFll) return fail(c, STARSIM_EINVAL, "n * tiles-per-star >= 2^32 (pair counts are 32-bit)");
  const size_t zbytes = sizeof(Header) + sizeof(uint32_t) * (CNT_STRIDE + 1) * (size_t)ntiles;
  // partial-tile buffers for split heavy tiles (a fixed count, so that the split -- and the summation order -- of a
  // tile is the same in a band render and in the full frame)
  const int part_cap = PART_CAP;
  int rc;
  if ((rc = grow(c, c->rec, sizeof(StarRec) * (size_t)(n > 0 ? n : 1), "records"))) return rc;
  const bool old_bins = !dbin_ok(fp, ntiles);  // bin.cu's pipeline needs the slot and sort scratch
  if (old_bins && (rc = grow(c, c->slots, sizeof(uint32_t) * (size_t)(pmax > 0 ? pmax : 1), "tile slots"))) return rc;
  if ((rc = grow(c, c->ids, sizeof(uint32_t) * (size_t)(pmax > 0 ? pmax : 1), "tile lists"))) return rc;
  if (old_bins && (rc = grow(c, c->tmp, sizeof(uint32_t) * (size_t)(pmax > 0 ? pmax : 1), "sort scratch"))) return rc;
  if ((rc = grow(c, c->tile_off, sizeof(uint32_t) * (size_t)(ntiles + 1), "tile offsets"))) return rc;
  if ((rc = grow(c, c->zeroed, zbytes, "header+counters"))) return rc;
  if ((rc = grow(c, c->items, sizeof(WorkItem) * (size_t)(ntiles + part_cap), "work items"))) return rc;
  if ((rc = grow(c, c->split_tab, sizeof(uint2) * (size_t)ntiles, "split table"))) return rc;
  if ((rc = grow(c, c->partial, sizeof(uint4) * (size_t)((ntiles + SCAN_TILES - 1) / SCAN_TILES), "scan partials")))
    return rc;
  if ((rc = grow(c, c->parts, sizeof(float) * TILE_W * TILE_H * (size_t)part_cap, "partial tiles"))) return rc;
  // segment scratch: one tile per persistent CTA of the tile kernels, one per tile for the sparse path
  if ((rc = grow(c, c->segs,
                 sizeof(float) * std::max<size_t>(tile8_scratch_floats(c->num_sms),
                                                  sparse ? (size_t)ntiles * TILE_W * TILE_H : 0),
                 "segment scratch")))
    return rc;
  if (ws_presort(c, fp)) {  // k_chsort's outputs
    if ((rc = grow(c, c->srec, sizeof(StarRec) * (size_t)(pmax > 0 ? pmax : 1), "bin-sorted records"))) return rc;
    if ((rc = grow(c, c->cbin, sizeof(uint16_t) * chsort_slots(ntiles, pmax) * chsort_words16(), "chunk bin starts")))
      return rc;
  }
  if (fp.tile_impl == STARSIM_TILE_T8 && R <= SB_MAXR) {  // k_t8sort's outputs (the t8 kernel only)
    if ((rc = grow(c, c->srec, sizeof(StarRec) * (size_t)(pmax > 0 ? pmax : 1), "bin-sorted records"))) return rc;
    if ((rc = grow(c, c->sbin, sizeof(uint32_t) * tile8_sbin_words(ntiles, part_cap, pmax), "segment bin starts")))
      return rc;
    if ((rc = grow(c, c->sext, sizeof(uint32_t) * (size_t)(ntiles + part_cap), "segment rows"))) return rc;
  }
  if (dbin_ok(fp, ntiles) &&
      (rc = grow(c, c->cmat, sizeof(uint32_t) * (size_t)ntiles * (size_t)(dbin_ctas(n) > 0 ? dbin_ctas(n) : 1),
                 "count matrix")))
    return rc;
  if ((dbin_ok(fp, ntiles) || sparse) &&
      (rc = grow(c, c->codes, sizeof(uint32_t) * (size_t)(n > 0 ? n : 1), "tile boxes")))
    return rc;
  if ((rc = grow(c, c->gbar, 64, "grid barrier"))) return rc;

  GraphKey key{x, y, mag, out, fp.n_dev, n, W, H, row0, rows, R, obits, c->psf | c->roi << 1, c->tile_impl, c->bin_impl, fp.ndst, {}, sigma, gain, st,
               c->scratch_gen};
  for (int i = 0; i < MAX_DST; ++i) key.dst[i] = fp.dst[i];
  if (st == nullptr || c->prof || !c->use_graphs) {
    if ((rc = enqueue_tiled(c, x, y, mag, n, fp, ntiles, tps, part_cap, out, st, sparse))) return rc;
  } else {
    if (!(c->have_graph && c->gkey == key)) {
      if (c->have_graph) {
        cudaGraphExecDestroy(c->gexec);
        c->have_graph = false;
      }
      cudaError_t e = cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal);
      if (e != cudaSuccess) return cuda_fail(c, e, "cudaStreamBeginCapture");
      rc = enqueue_tiled(c, x, y, mag, n, fp, ntiles, tps, part_cap, out, st, sparse);
      cudaGraph_t graph = nullptr;
      e = cudaStreamEndCapture(st, &graph);
      if (rc) {
        if (graph) cudaGraphDestroy(graph);
        return rc;
      }
      if (e != cudaSuccess) return cuda_fail(c, e, "cudaStreamEndCapture");
      e = cudaGraphInstantiate(&c->gexec, graph, 0);
      cudaGraphDestroy(graph);
      if (e != cudaSuccess) return cuda_fail(c, e, "cudaGraphInstantiate");
      c->gkey = key;
      c->have_graph = true;
    }
    cudaError_t e = cudaGraphLaunch(c->gexec, st);
    if (e != cudaSuccess) return cuda_fail(c, e, "cudaGraphLaunch");
  }
  c->have_bins = true;
  c->last_stream = st;
  c->last_ntiles = ntiles;
  c->last_sparse = sparse;
  if (sparse) c->sp = {x, y, mag, n, fp, tps, part_cap};
  c->err.clear();
  return STARSIM_OK;
}

}  // namespace

extern "C" {

int starsim_create(starsim_ctx** out, int cuda_device) {
  if (!out) {
    g_create_error = "out is NULL";
    return STARSIM_EINVAL;
  }
  *out = nullptr;
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    g_create_error = std::string("no CUDA device: ") + cudaGetErrorString(e);
    return STARSIM_ENODEV;
  }
  if (cuda_device < 0 || cuda_device >= ndev) {
    g_create_error = "cuda_device out of range";
    return STARSIM_EINVAL;
  }
  cudaDeviceProp prop;
  if ((e = cudaGetDeviceProperties(&prop, cuda_device)) != cudaSuccess) {
    g_create_error = std::string("cudaGetDeviceProperties: ") + cudaGetErrorString(e);
    return STARSIM_ECUDA;
  }
  if (!(prop.major == 10 && prop.minor == 0)) {
    g_create_error = std::string("device ") + prop.name + " is sm_" + std::to_string(prop.major) +
                     std::to_string(prop.minor) + "; libstarsim.so carries sm_100a code only";
    return STARSIM_ENODEV;
  }
  starsim_ctx* c = new starsim_ctx();
  c->dev = cuda_device;
  c->num_sms = prop.multiProcessorCount;
  init_kernels();
  // k_dfused (one cooperative launch for the three binning kernels) is opt-in: STARSIM_DFUSED=1 at context creation
  // (same CSR; measured 2-6 us slower per frame than the three graph-replayed kernels)
  const char* df = getenv("STARSIM_DFUSED");
  c->dfused_grid = (df && df[0] == '1') ? dfused_max_grid(c->num_sms) : 0;
  const char* wp = getenv("STARSIM_WS_PRESORT");
  c->ws_presort = wp && wp[0] == '1';
  const char* ng = getenv("STARSIM_NO_GRAPH");
  c->use_graphs = !(ng && ng[0] == '1');
  *out = c;
  g_create_error.clear();
  return STARSIM_OK;
}

void starsim_destroy(starsim_ctx* c) {
  if (!c) return;
  {
    DevGuard g(c->dev);
    cudaDeviceSynchronize();
    if (c->have_graph) cudaGraphExecDestroy(c->gexec);
    Buf* bufs[] = {&c->rec, &c->slots, &c->ids, &c->tmp, &c->tile_off, &c->items, &c->split_tab, &c->parts,
                   &c->partial, &c->zeroed, &c->stage, &c->cmat, &c->codes, &c->segs, &c->srec, &c->sbin, &c->sext,
                   &c->rblk, &c->cbin, &c->gbar};
    for (Buf* b : bufs)
      if (b->p) cudaFree(b->p);
    for (auto& l : c->pending) {
      cudaEventDestroy(l.a);
      cudaEventDestroy(l.b);
    }
    for (cudaEvent_t e : c->ev_pool) cudaEventDestroy(e);
  }
  delete c;
}

const char* starsim_last_error(const starsim_ctx* c) { return c ? c->err.c_str() : g_create_error.c_str(); }

int starsim_render(starsim_ctx* c, const float* x, const float* y, const float* mag, int64_t n, int32_t W, int32_t H,
                   float sigma, int32_t R, float gain, float* out, starsim_stream_t stream) {
  if (!c) return STARSIM_EINVAL;
  int rc = validate_frame(c, x, y, mag, n, W, H, sigma, R, gain, out);
  if (rc) return rc;
  return render_tiled(c, x, y, mag, n, W, H, 0, H, sigma, R, gain, 0, out, (cudaStream_t)stream);
}

int starsim_render_band(starsim_ctx* c, const float* x, const float* y, const float* mag, int64_t n, int32_t W,
                        int32_t H, int32_t row0, int32_t rows, float sigma, int32_t R, float gain, float* out_band,
                        starsim_stream_t stream) {
  if (!c) return STARSIM_EINVAL;
  int rc = validate_frame(c, x, y, mag, n, W, H, sigma, R, gain, out_band);
  if (rc) return rc;
  if (row0 < 0 || rows < 1 || (int64_t)row0 + rows > H) return fail(c, STARSIM_EINVAL, "band not inside the image");
  return render_tiled(c, x, y, mag, n, W, H, row0, rows, sigma, R, gain, 0, out_band, (cudaStream_t)stream);
}

int starsim_render_band_to(starsim_ctx* c, const float* x, const float* y, const float* mag, int64_t n, int32_t W,
                           int32_t H, int32_t row0, int32_t rows, float sigma, int32_t R, float gain,
                           float* const* dsts, int32_t ndst, starsim_stream_t stream) {
  if (!c) return STARSIM_EINVAL;
  if (!dsts || ndst < 1 || ndst > MAX_DST) return fail(c, STARSIM_EINVAL, "ndst outside [1, 8] or dsts NULL");
  for (int i = 0; i < ndst; ++i)
    if (!dsts[i]) return fail(c, STARSIM_EINVAL, "NULL destination frame");
  int rc = validate_frame(c, x, y, mag, n, W, H, sigma, R, gain, dsts[0]);
  if (rc) return rc;
  if (row0 < 0 || rows < 1 || (int64_t)row0 + rows > H) return fail(c, STARSIM_EINVAL, "band not inside the image");
  return render_tiled(c, x, y, mag, n, W, H, row0, rows, sigma, R, gain, 0, dsts[0] + (int64_t)row0 * W,
                      (cudaStream_t)stream, dsts, ndst);
}

int starsim_render_gray(starsim_ctx* c, const float* x, const float* y, const float* mag, int64_t n, int32_t W,
                        int32_t H, float sigma, int32_t R, float gain, int32_t bits, void* out,
                        starsim_stream_t stream) {
  if (!c) return STARSIM_EINVAL;
  int rc = validate_frame(c, x, y, mag, n, W, H, sigma, R, gain, out);
  if (rc) return rc;
  if (bits != 8 && bits != 16) return fail(c, STARSIM_EINVAL, "bits must be 8 or 16");
  return render_tiled(c, x, y, mag, n, W, H, 0, H, sigma, R, gain, bits, out, (cudaStream_t)stream);
}

int starsim_set_psf(starsim_ctx* c, int32_t mode) {
  if (!c) return STARSIM_EINVAL;
  if (mode != STARSIM_PSF_POINT && mode != STARSIM_PSF_INTEGRATED)
    return fail(c, STARSIM_EINVAL, "psf mode must be STARSIM_PSF_POINT or STARSIM_PSF_INTEGRATED");
  c->psf = mode;
  c->err.clear();
  return STARSIM_OK;
}

int starsim_set_roi(starsim_ctx* c, int32_t shape) {
  if (!c) return STARSIM_EINVAL;
  if (shape != STARSIM_ROI_SQUARE && shape != STARSIM_ROI_CIRCLE)
    return fail(c, STARSIM_EINVAL, "roi shape must be STARSIM_ROI_SQUARE or STARSIM_ROI_CIRCLE");
  c->roi = shape;
  c->err.clear();
  return STARSIM_OK;
}

int starsim_set_binning(starsim_ctx* c, int32_t mode) {
  if (!c) return STARSIM_EINVAL;
  if (mode != STARSIM_BIN_AUTO && mode != STARSIM_BIN_ATOMIC)
    return fail(c, STARSIM_EINVAL, "binning mode must be STARSIM_BIN_AUTO or STARSIM_BIN_ATOMIC");
  c->bin_impl = mode;
  c->err.clear();
  return STARSIM_OK;
}

int starsim_set_star_count(starsim_ctx* c, const uint32_t* n_dev) {
  if (!c) return STARSIM_EINVAL;
  c->n_dev = n_dev;
  c->err.clear();
  return STARSIM_OK;
}

int starsim_route_band(starsim_ctx* c, const float* x, const float* y, const float* mag, int64_t n, int32_t H,
                       int32_t row0, int32_t rows, int32_t R, float* x_out, float* y_out, float* mag_out,
                       uint32_t* n_out, starsim_stream_t stream) {
  if (!c) return STARSIM_EINVAL;
  if (n < 0) return fail(c, STARSIM_EINVAL, "n < 0");
  if (n > 0xFFFFFFFFll) return fail(c, STARSIM_EINVAL, "n >= 2^32 (star indices are 32-bit)");
  if (n > 0 && (!x || !y || !mag || !x_out || !y_out || !mag_out))
    return fail(c, STARSIM_EINVAL, "n > 0 with a NULL input or output array");
  if (!n_out) return fail(c, STARSIM_EINVAL, "n_out is NULL");
  if (H < 1 || H > STARSIM_MAX_DIM) return fail(c, STARSIM_EINVAL, "height outside [1, 32767]");
  if (row0 < 0 || rows < 1 || (int64_t)row0 + rows > H) return fail(c, STARSIM_EINVAL, "band not inside the image");
  if (R < 1 || R > STARSIM_MAX_ROI) return fail(c, STARSIM_EINVAL, "roi outside [1, 255]");
  DevGuard g(c->dev);
  cudaStream_t st = (cudaStream_t)stream;
  int rc;
  if ((rc = grow(c, c->rblk, sizeof(uint32_t) * (route_blocks(n) > 0 ? route_blocks(n) : 1), "route blocks")))
    return rc;
  timed(
      c, 8, st,
      [&] {
        launch_route(x, y, mag, n, row0, rows, R, (uint32_t*)c->rblk.p, x_out, y_out, mag_out, n_out, st);
      },
      n > 0 ? 2 : 1);
  if ((rc = check_launch(c, "k_route"))) return rc;
  c->err.clear();
  return STARSIM_OK;
}

int starsim_set_tile_kernel(starsim_ctx* c, int32_t mode) {
  if (!c) return STARSIM_EINVAL;
  if (mode != STARSIM_TILE_AUTO && mode != STARSIM_TILE_LISTS && mode != STARSIM_TILE_SB && mode != STARSIM_TILE_WS &&
      mode != STARSIM_TILE_T8)
    return fail(c, STARSIM_EINVAL, "tile kernel mode must be STARSIM_TILE_AUTO, _LISTS, _SB, _WS or _T8");
  c->tile_impl = mode;
  c->err.clear();
  return STARSIM_OK;
}

int starsim_render_atomic(starsim_ctx* c, const float* x, const float* y, const float* mag, int64_t n, int32_t W,
                          int32_t H, float sigma, int32_t R, float gain, float* out, starsim_stream_t stream) {
  if (!c) return STARSIM_EINVAL;
  int rc = validate_frame(c, x, y, mag, n, W, H, sigma, R, gain, out);
  if (rc) return rc;
  if (c->n_dev) return fail(c, STARSIM_EINVAL, "a device star count (starsim_set_star_count) is set: tiled renders only");
  DevGuard g(c->dev);
  cudaStream_t st = (cudaStream_t)stream;
  FrameParams fp = make_params(W, H, 0, H, sigma, R, gain, c->psf);
  fp.roi = c->roi;
  timed(c, 5, st, [&] { cudaMemsetAsync(out, 0, sizeof(float) * (size_t)W * H, st); });
  timed(c, 4, st, [&] { launch_atomic(x, y, mag, n, fp, out, st); });
  if ((rc = check_launch(c, "k_atomic"))) return rc;
  c->err.clear();
  return STARSIM_OK;
}

int starsim_render_lut(starsim_ctx* c, const float* x, const float* y, const float* mag, int64_t n, int32_t W,
                       int32_t H, float sigma, int32_t R, float gain, float* out, starsim_stream_t stream) {
  if (!c) return STARSIM_EINVAL;
  int rc = validate_frame(c, x, y, mag, n, W, H, sigma, R, gain, out);
  if (rc) return rc;
  if (R > STARSIM_MAX_LUT_ROI) return fail(c, STARSIM_EINVAL, "roi > 63 for the lookup-table kernel");
  if (c->n_dev) return fail(c, STARSIM_EINVAL, "a device star count (starsim_set_star_count) is set: tiled renders only");
  DevGuard g(c->dev);
  cudaStream_t st = (cudaStream_t)stream;
  FrameParams fp = make_params(W, H, 0, H, sigma, R, gain, c->psf);
  fp.roi = c->roi;
  timed(c, 5, st, [&] { cudaMemsetAsync(out, 0, sizeof(float) * (size_t)W * H, st); });
  timed(c, 4, st, [&] { launch_lut(x, y, mag, n, fp, out, st); });
  if ((rc = check_launch(c, "k_lut"))) return rc;
  c->err.clear();
  return STARSIM_OK;
}

int starsim_upload_aos(starsim_ctx* c, const void* host_aos, int64_t n, float* x, float* y, float* mag,
                       starsim_stream_t stream) {
  if (!c) return STARSIM_EINVAL;
  if (n < 0) return fail(c, STARSIM_EINVAL, "n < 0");
  if (n == 0) return STARSIM_OK;
  if (!host_aos || !x || !y || !mag) return fail(c, STARSIM_EINVAL, "NULL pointer with n > 0");
  DevGuard g(c->dev);
  cudaStream_t st = (cudaStream_t)stream;
  int rc = grow(c, c->stage, sizeof(float) * 3 * (size_t)n, "aos staging");
  if (rc) return rc;
  cudaError_t e = cudaMemcpyAsync(c->stage.p, host_aos, sizeof(float) * 3 * (size_t)n, cudaMemcpyHostToDevice, st);
  if (e != cudaSuccess) return cuda_fail(c, e, "cudaMemcpyAsync(aos)");
  timed(c, 7, st, [&] { launch_split_aos((const float*)c->stage.p, n, x, y, mag, c->num_sms, st); });
  if ((rc = check_launch(c, "k_split_aos"))) return rc;
  c->err.clear();
  return STARSIM_OK;
}

int starsim_quantize(starsim_ctx* c, const float* img, int64_t npix, int32_t bits, void* out,
                     starsim_stream_t stream) {
  if (!c) return STARSIM_EINVAL;
  if (npix < 0) return fail(c, STARSIM_EINVAL, "npix < 0");
  if (bits != 8 && bits != 16) return fail(c, STARSIM_EINVAL, "bits must be 8 or 16");
  if (npix > 0 && (!img || !out)) return fail(c, STARSIM_EINVAL, "NULL pointer with npix > 0");
  if (npix == 0) return STARSIM_OK;
  DevGuard g(c->dev);
  cudaStream_t st = (cudaStream_t)stream;
  timed(c, 6, st, [&] { launch_quantize(img, npix, bits, out, c->num_sms, st); });
  int rc = check_launch(c, "k_quantize");
  if (rc) return rc;
  c->err.clear();
  return STARSIM_OK;
}

int starsim_get_bins(starsim_ctx* c, int32_t* tile_w, int32_t* tile_h, uint32_t* tile_off_host, int64_t off_cap,
                     uint32_t* ids_host, int64_t ids_cap, int64_t* n_pairs) {
  if (!c) return STARSIM_EINVAL;
  if (!c->have_bins) return fail(c, STARSIM_EINVAL, "no tiled render on this ctx yet");
  DevGuard g(c->dev);
  if (c->last_sparse) {
    // the last render took the sparse path: bin its (still caller-owned) arrays now, on its stream
    const bool prof = c->prof;
    c->prof = false;
    const int rc = enqueue_binning(c, c->sp.x, c->sp.y, c->sp.m, c->sp.n, c->sp.fp, c->last_ntiles, c->sp.tps,
                                   c->sp.part_cap, c->last_stream);
    c->prof = prof;
    if (rc) return rc;
    c->last_sparse = false;
  }
  cudaError_t e = cudaStreamSynchronize(c->last_stream);
  if (e != cudaSuccess) return cuda_fail(c, e, "cudaStreamSynchronize");
  Header h;
  if ((e = cudaMemcpy(&h, c->zeroed.p, sizeof(Header), cudaMemcpyDeviceToHost)) != cudaSuccess)
    return cuda_fail(c, e, "cudaMemcpy(header)");
  if (tile_w) *tile_w = TILE_W;
  if (tile_h) *tile_h = TILE_H;
  if (n_pairs) *n_pairs = h.P;
  if (off_cap < c->last_ntiles + 1 || ids_cap < (int64_t)h.P || !tile_off_host || (!ids_host && h.P))
    return fail(c, STARSIM_EINVAL, "capacity too small (need ntiles+1 offsets and P ids)");
  if ((e = cudaMemcpy(tile_off_host, c->tile_off.p, sizeof(uint32_t) * (size_t)(c->last_ntiles + 1),
                      cudaMemcpyDeviceToHost)) != cudaSuccess)
    return cuda_fail(c, e, "cudaMemcpy(tile_off)");
  if (h.P && (e = cudaMemcpy(ids_host, c->ids.p, sizeof(uint32_t) * h.P, cudaMemcpyDeviceToHost)) != cudaSuccess)
    return cuda_fail(c, e, "cudaMemcpy(ids)");
  c->err.clear();
  return STARSIM_OK;
}

int starsim_profile(starsim_ctx* c, int enable) {
  if (!c) return STARSIM_EINVAL;
  DevGuard g(c->dev);
  for (auto& l : c->pending) {
    cudaEventSynchronize(l.b);
    c->ev_pool.push_back(l.a);
    c->ev_pool.push_back(l.b);
  }
  c->pending.clear();
  for (int k = 0; k < STARSIM_NUM_KCLASS; ++k) {
    c->ms[k] = 0;
    c->launches[k] = 0;
  }
  c->prof = enable != 0;
  return STARSIM_OK;
}

int starsim_kernel_times(starsim_ctx* c, double* ms, int64_t* launches) {
  if (!c) return STARSIM_EINVAL;
  if (!ms || !launches) return fail(c, STARSIM_EINVAL, "NULL output array");
  DevGuard g(c->dev);
  for (auto& l : c->pending) {
    cudaError_t e = cudaEventSynchronize(l.b);
    if (e != cudaSuccess) return cuda_fail(c, e, "cudaEventSynchronize");
    float t = 0;
    cudaEventElapsedTime(&t, l.a, l.b);
    c->ms[l.kclass] += t;
    c->launches[l.kclass] += l.n;
    c->ev_pool.push_back(l.a);
    c->ev_pool.push_back(l.b);
  }
  c->pending.clear();
  for (int k = 0; k < STARSIM_NUM_KCLASS; ++k) {
    ms[k] = c->ms[k];
    launches[k] = c->launches[k];
  }
  return STARSIM_OK;
}

}  // extern "C"
