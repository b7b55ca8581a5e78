"""Random-row-gather ceiling ("a measured random-row-gather
ceiling"): the HBM read bandwidth of gathering uniformly random rows of a
SIFT1M-sized table (1M x 128 fp32, 512 B rows) — the search's access pattern
without its dependency chains.  A probe kernel (JIT-compiled here for sm_100a;
measurement tooling, not the product path): each warp reads 8 random rows per
round with 16 B per lane (all in flight), folds them into a checksum, grid =
148 SMs x 16 warps x 4; CUDA events, L2 flushed before each run.  Also a table
larger than L2 read sequentially, and 128 B rows (the adjacency rows).

    python tools/gather_ceiling.py [--out gpurun_out/gather_ceiling.json]
"""
import argparse
import json
import os

SRC = r"""
#include <cstdint>
__global__ void gather_rows(const float4* __restrict__ x, int row_f4, const int* __restrict__ idx,
                            long long n_idx, float* out) {
  const int lane = threadIdx.x & 31;
  const long long w = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  float acc = 0.f;
  for (long long base = w * 8; base < n_idx; base += nw * 8) {
    float4 v[8];
#pragma unroll
    for (int r = 0; r < 8; ++r) {
      const long long k = base + r;
      const int id = k < n_idx ? __ldg(idx + k) : 0;
      v[r] = (lane < row_f4 && k < n_idx) ? __ldcs(x + (long long)id * row_f4 + lane)
                                          : make_float4(0.f, 0.f, 0.f, 0.f);
    }
#pragma unroll
    for (int r = 0; r < 8; ++r) acc += v[r].x + v[r].y + v[r].z + v[r].w;
  }
  if (acc == 1234.5f) out[0] = acc;  // keep the loads
}
void launch(torch::Tensor x, int row_f4, torch::Tensor idx, torch::Tensor out, int grid) {
  gather_rows<<<grid, 512>>>(reinterpret_cast<const float4*>(x.data_ptr<float>()), row_f4,
                             idx.data_ptr<int>(), idx.numel(), out.data_ptr<float>());
}
"""


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default="gpurun_out/gather_ceiling.json")
    a = ap.parse_args()
    import torch
    from torch.utils.cpp_extension import load_inline
    mod = load_inline("gather_ceiling", cpp_sources="void launch(torch::Tensor x, int row_f4, torch::Tensor idx, torch::Tensor out, int grid);",
                      cuda_sources="#include <torch/extension.h>\n" + SRC, functions=["launch"],
                      extra_cuda_cflags=["-gencode", "arch=compute_100a,code=sm_100a", "-O3"],
                      verbose=False)
    dev = torch.device("cuda", 0)
    sms = torch.cuda.get_device_properties(dev).multi_processor_count
    g = torch.Generator(device=dev).manual_seed(0)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    out = torch.zeros(1, device=dev)
    res = {"probe": "8 rows in flight per warp, 16 B per lane, grid = SMs x 4 CTAs x 16 warps"}
    cases = [("rows512B_uniform_1M", 1_000_000, 128, "uniform"),
             ("rows512B_uniform_16M", 16_000_000, 128, "uniform"),
             ("rows128B_uniform_1M", 1_000_000, 32, "uniform"),
             ("rows512B_sequential_16M", 16_000_000, 128, "seq")]
    for name, rows, dim, kind in cases:
        x = torch.randn(rows, dim, device=dev)
        n_idx = 16_000_000
        idx = (torch.randint(0, rows, (n_idx,), device=dev, generator=g, dtype=torch.int32)
               if kind == "uniform" else (torch.arange(n_idx, device=dev) % rows).int())
        ts = []
        for i in range(8):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            mod.launch(x, dim // 4, idx, out, sms * 4)
            e1.record()
            torch.cuda.synchronize()
            if i >= 2:
                ts.append(e0.elapsed_time(e1))
        ms = min(ts)
        res[name] = {"ms": round(ms, 4), "row_bytes": dim * 4,
                     "read_GBps": round(n_idx * dim * 4 / ms / 1e6, 1)}
        print(name, res[name], flush=True)
        del x, idx
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
