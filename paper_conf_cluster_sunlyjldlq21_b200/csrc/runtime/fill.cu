// fill.cu — device twin of the cstgen input generator (cstgen/cst_gen.h).
// Fills the logical padded region of a grid with U[-1,1) values keyed by the GLOBAL padded
// index, so any rank can generate its own slab (and its halo) without the global array.
#include "../../../cstgen/cst_gen.h"
#include "internal.h"

namespace {

__global__ void fill_kernel(double* __restrict__ dst, int64_t nx, int64_t ny, int64_t nz,
                            int64_t halo, int64_t lead_x, int64_t pitch_x, int64_t pitch_y,
                            uint64_t key, int64_t nxg, int64_t nyg, int64_t z0, double pad) {
  const int64_t row = blockIdx.x;  // (z, y) row of the allocation
  const int64_t planes = nz + 2 * halo;
  const int64_t zz = row / pitch_y, yy = row % pitch_y;
  if (zz >= planes) return;
  const int64_t y = yy - halo, z = zz - halo;
  double* r = dst + row * pitch_x;
  const bool row_in = y < ny + halo;
  for (int64_t xx = threadIdx.x; xx < pitch_x; xx += blockDim.x) {
    const int64_t x = xx - lead_x;
    double v = pad;
    if (row_in && x >= -halo && x < nx + halo)
      v = cstgen_value(key, cstgen_index(nxg, nyg, halo, x, y, z + z0));
    r[xx] = v;
  }
}

// one warp per (z, y) row of the logical padded region [-halo, n + halo)^3: halo rows are
// copied whole, interior rows only their 2*halo x-halo elements.  A z-halo plane that faces
// a z-slab neighbour (zlo / zhi = 0) is treated like an interior plane: its x/y ring is
// copied, its interior x/y is the exchange's (the neighbour's stores or NCCL receive)
__global__ void copy_halo_kernel(const double* __restrict__ src, double* __restrict__ dst,
                                 int64_t nx, int64_t ny, int64_t nz, int64_t halo,
                                 int64_t lead_x, int64_t pitch_x, int64_t pitch_y, int zlo,
                                 int zhi) {
  const int64_t row = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / 32;
  const int lane = threadIdx.x % 32;
  const int64_t rows_y = ny + 2 * halo;
  if (row >= rows_y * (nz + 2 * halo)) return;
  const int64_t y = row % rows_y - halo, z = row / rows_y - halo;
  const bool facing = (z < 0 && !zlo) || (z >= nz && !zhi);
  const int64_t base = ((z + halo) * pitch_y + (y + halo)) * pitch_x + lead_x;
  if (y < 0 || y >= ny || ((z < 0 || z >= nz) && !facing)) {
    for (int64_t x = lane - halo; x < nx + halo; x += 32) dst[base + x] = src[base + x];
  } else if (lane < 2 * halo) {
    const int64_t x = lane < halo ? lane - halo : nx + (lane - halo);
    dst[base + x] = src[base + x];
  }
}

}  // namespace

namespace cst {
// Copy the logical halo of one array (the multi-step boundary condition) from src to dst;
// zlo / zhi = false: the z-halo planes on that side face a z-slab neighbour, only their x/y
// ring is copied.
cst_status copy_halo(const cst_grid& g, const double* src, double* dst, cudaStream_t stream,
                     bool zlo, bool zhi) {
  const int64_t rows = (g.nz + 2 * (int64_t)g.halo) * (g.ny + 2 * (int64_t)g.halo);
  if (g.halo > 16) return fail(CST_E_UNSUPPORTED, "copy_halo: halo > 16");
  const int64_t blocks = (rows * 32 + 255) / 256;
  if (blocks > 0x7fffffffLL) return fail(CST_E_UNSUPPORTED, "grid too large for copy_halo");
  copy_halo_kernel<<<(unsigned)blocks, 256, 0, stream>>>(src, dst, g.nx, g.ny, g.nz, g.halo,
                                                         g.lead_x, g.pitch_x, g.pitch_y,
                                                         zlo ? 1 : 0, zhi ? 1 : 0);
  CST_CUDA(cudaGetLastError());
  return CST_OK;
}
}  // namespace cst

extern "C" cst_status cst_fill_uniform(const cst_grid* g, double* dev, uint64_t seed,
                                       uint64_t array_id, int64_t nx_global, int64_t ny_global,
                                       int64_t z0, double pad_value, void* stream) {
  if (!g || !dev) return cst::fail(CST_E_INVALID, "null argument");
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess || n == 0) {
    cudaGetLastError();
    return cst::fail(CST_E_CUDA, "no CUDA device available (libcst has no CPU fallback)");
  }
  const int64_t rows = (g->nz + 2 * (int64_t)g->halo) * g->pitch_y;
  if (rows > 0x7fffffffLL) return cst::fail(CST_E_UNSUPPORTED, "grid too large for fill");
  fill_kernel<<<(unsigned)rows, 256, 0, (cudaStream_t)stream>>>(
      dev, g->nx, g->ny, g->nz, g->halo, g->lead_x, g->pitch_x, g->pitch_y,
      cstgen_key(seed, array_id), nx_global, ny_global, z0, pad_value);
  CST_CUDA(cudaGetLastError());
  return CST_OK;
}
