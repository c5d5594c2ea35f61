// synth_gen.cu -- device generator of the config-5 mesh batch (INPUT GENERATION
// ONLY: no arithmetic of the RCM method).  Reproduces synth.c5_matrix(k, N)
// bit-exactly: a 2D 5-point (even k) or 3D 27-point (odd k) grid with stored
// diagonal, relabelled by the counter-based Feistel permutation of
// synth.randperm(n, 50000 + k), rows sorted ascending.
#include <cstdint>
#include <cuda_runtime.h>

namespace {

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

struct Feistel {
  uint64_t key[4];
  uint64_t mask;
  int h;
  uint64_t n;
  __device__ void init(uint64_t nn, uint64_t seed) {
    n = nn;
    int b = 2;
    uint64_t m = nn > 2 ? nn - 1 : 1;
    int bl = 64 - __clzll((long long)m);
    b = bl > 2 ? bl : 2;
    b += b & 1;
    h = b / 2;
    mask = (1ull << h) - 1;
    for (int r = 0; r < 4; ++r) key[r] = mix64((seed * 4 + r + 1) * 0x9E3779B97F4A7C15ull);
  }
  __device__ uint64_t enc1(uint64_t x) const {
    uint64_t l = (x >> h) & mask, r = x & mask;
    for (int i = 0; i < 4; ++i) {
      uint64_t f = mix64(r ^ key[i]) & mask;
      uint64_t t = r;
      r = l ^ f;
      l = t;
    }
    return (l << h) | r;
  }
  __device__ uint64_t dec1(uint64_t y) const {
    uint64_t l = (y >> h) & mask, r = y & mask;
    for (int i = 3; i >= 0; --i) {
      uint64_t ol = r ^ (mix64(l ^ key[i]) & mask);
      r = l;
      l = ol;
    }
    return (l << h) | r;
  }
  __device__ uint64_t fwd(uint64_t x) const {   // cycle-walked image
    uint64_t y = enc1(x);
    while (y >= n) y = enc1(y);
    return y;
  }
  __device__ uint64_t inv(uint64_t y) const {
    uint64_t x = dec1(y);
    while (x >= n) x = dec1(x);
    return x;
  }
};

struct MatSpec {           // per matrix
  int32_t kind;            // 2 = 2D 5-point, 3 = 3D 27-point
  int32_t nx, ny, nz;
  int32_t gid;             // global matrix index k (relabel seed 50000 + k)
};

__device__ int find_mat(const int64_t* node_off, int num, long long g) {
  int lo = 0, hi = num - 1;
  while (lo < hi) {
    int mid = (lo + hi + 1) >> 1;
    if (node_off[mid] <= g) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// neighbours (old ids, ascending, diagonal included) of old node v
__device__ int stencil(const MatSpec& s, int v, int* nb) {
  int c = 0;
  if (s.kind == 2) {
    const int w = s.nx, hgt = s.ny;
    const int x = v % w, y = v / w;
    if (y > 0) nb[c++] = v - w;
    if (x > 0) nb[c++] = v - 1;
    nb[c++] = v;
    if (x < w - 1) nb[c++] = v + 1;
    if (y < hgt - 1) nb[c++] = v + w;
    return c;
  }
  const int nx = s.nx, ny = s.ny, nz = s.nz;
  const int x = v % nx, y = (v / nx) % ny, z = v / (nx * ny);
  for (int dz = -1; dz <= 1; ++dz)
    for (int dy = -1; dy <= 1; ++dy)
      for (int dx = -1; dx <= 1; ++dx) {
        if (x + dx < 0 || x + dx >= nx || y + dy < 0 || y + dy >= ny || z + dz < 0 || z + dz >= nz) continue;
        nb[c++] = v + (dz * ny + dy) * nx + dx;
      }
  return c;
}

__global__ void k_degrees(const MatSpec* __restrict__ specs, const int64_t* __restrict__ node_off, int num,
                          long long total, int32_t* __restrict__ deg) {
  for (long long g = blockIdx.x * (long long)blockDim.x + threadIdx.x; g < total;
       g += (long long)gridDim.x * blockDim.x) {
    const int k = find_mat(node_off, num, g);
    const MatSpec s = specs[k];
    const int n = (int)(node_off[k + 1] - node_off[k]);
    Feistel f;
    f.init((uint64_t)n, 50000ull + (uint64_t)s.gid);
    const int u = (int)(g - node_off[k]);
    const int v = n > 1 ? (int)f.inv((uint64_t)u) : 0;
    int nb[27];
    deg[g] = stencil(s, v, nb);
  }
}

__global__ void k_fill(const MatSpec* __restrict__ specs, const int64_t* __restrict__ node_off,
                       const int64_t* __restrict__ nnz_off, int num, long long total,
                       const int32_t* __restrict__ rp_local, int32_t* __restrict__ col) {
  for (long long g = blockIdx.x * (long long)blockDim.x + threadIdx.x; g < total;
       g += (long long)gridDim.x * blockDim.x) {
    const int k = find_mat(node_off, num, g);
    const MatSpec s = specs[k];
    const int n = (int)(node_off[k + 1] - node_off[k]);
    Feistel f;
    f.init((uint64_t)n, 50000ull + (uint64_t)s.gid);
    const int u = (int)(g - node_off[k]);
    const int v = n > 1 ? (int)f.inv((uint64_t)u) : 0;
    int nb[27];
    const int d = stencil(s, v, nb);
    for (int i = 0; i < d; ++i) nb[i] = n > 1 ? (int)f.fwd((uint64_t)nb[i]) : 0;
    for (int i = 1; i < d; ++i) {   // insertion sort (<= 27)
      int x = nb[i], j = i - 1;
      while (j >= 0 && nb[j] > x) { nb[j + 1] = nb[j]; --j; }
      nb[j + 1] = x;
    }
    int32_t* out = col + nnz_off[k] + rp_local[g + k];
    for (int i = 0; i < d; ++i) out[i] = nb[i];
  }
}

}  // namespace

extern "C" int synth_c5_degrees(const void* specs, const int64_t* node_off, int num, long long total,
                                int32_t* deg, void* stream) {
  const int blocks = (int)((total + 255) / 256 < 148 * 32 ? (total + 255) / 256 : 148 * 32);
  k_degrees<<<blocks, 256, 0, (cudaStream_t)stream>>>((const MatSpec*)specs, node_off, num, total, deg);
  return (int)cudaGetLastError();
}

extern "C" int synth_c5_fill(const void* specs, const int64_t* node_off, const int64_t* nnz_off, int num,
                             long long total, const int32_t* rp_local, int32_t* col, void* stream) {
  const int blocks = (int)((total + 255) / 256 < 148 * 32 ? (total + 255) / 256 : 148 * 32);
  k_fill<<<blocks, 256, 0, (cudaStream_t)stream>>>((const MatSpec*)specs, node_off, nnz_off, num, total,
                                                   rp_local, col);
  return (int)cudaGetLastError();
}
