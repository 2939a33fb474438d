// cells.cuh -- the cell of a position in a binning grid (k_bin.cu builds the
// sorted order; k_sym.cu looks agents up in it).
#pragma once
#include "internal.h"

namespace boids {

__device__ __forceinline__ uint32_t spread3(uint32_t x) {  // 10 bits -> every 3rd bit
  x &= 0x3ff;
  x = (x | (x << 16)) & 0x030000FF;
  x = (x | (x << 8)) & 0x0300F00F;
  x = (x | (x << 4)) & 0x030C30C3;
  x = (x | (x << 2)) & 0x09249249;
  return x;
}

__device__ __forceinline__ int cell_coord(float v, const BinGrid& g, int d) {
  // floor((v - lo) * inv_h), clamped into [0, dim-1]; NaN handled by the caller
  float t = (v - g.lo[d]) * g.inv_h;
  int c = (int)floorf(t);
  return c < 0 ? 0 : (c >= g.dim[d] ? g.dim[d] - 1 : c);
}

__device__ __forceinline__ int fine_coord(float v, const BinGrid& g, int d) {
  float t = (v - g.lo[d]) * g.inv_h;
  int c = (int)floorf(t);
  return c < 0 ? 0 : (c >= g.fdim[d] ? g.fdim[d] - 1 : c);
}

__device__ __forceinline__ int cell_of(float4 p, const BinGrid& g) {
  if (g.block > 0) {  // block of the fine cell (exactly the fine cell's own coordinates / block)
    const int bx = fine_coord(p.x, g, 0) / g.block, by = fine_coord(p.y, g, 1) / g.block,
              bz = fine_coord(p.z, g, 2) / g.block;
    return (bz * g.dim[1] + by) * g.dim[0] + bx;
  }
  int ix = cell_coord(p.x, g, 0), iy = cell_coord(p.y, g, 1), iz = cell_coord(p.z, g, 2);
  if (g.morton) return (int)(spread3(ix) | (spread3(iy) << 1) | (spread3(iz) << 2));
  return (iz * g.dim[1] + iy) * g.dim[0] + ix;
}

}  // namespace boids
