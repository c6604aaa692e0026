"""SURVEY §8(c) P3, B200 part: the paper's shared-memory occupancy formula
(Fig 12: max_blocks_by_shmem = min(floor(smem_SM /
shmem_per_block), max_blocks_per_multi_processor)) against the CUDA
occupancy calculator of the B200 itself, for a kernel whose only limiter is
its dynamic shared memory.

This documents the paper-vs-hardware gap of reading A11 (the 1 KB per-block
shared-memory reservation of sm_80+ is not modelled by Fig 12); it is not a
parity target: the oracle and the kernels follow Fig 12 literally.  The
calculator is reached through cuda-python (driver API + NVRTC); nothing here
touches the library or the oracle.
"""
from __future__ import annotations

import pytest

SMEM_SM = 233472          # B200 shared memory per SM (reading A10)
MAX_BLOCKS = 32           # cc 10.0 max resident blocks per SM (reading A10)
THREADS_SM = 2048


def _calculator():
    import torch
    from cuda.bindings import driver, nvrtc

    torch.zeros(1, device="cuda")        # primary context current on this thread
    src = (b'extern "C" __global__ void k(int *p) {\n'
           b'  extern __shared__ int s[];\n'
           b'  s[threadIdx.x] = threadIdx.x; __syncthreads();\n'
           b'  if (p) p[threadIdx.x] = s[(threadIdx.x + 1) % blockDim.x];\n}\n')
    err, prog = nvrtc.nvrtcCreateProgram(src, b"occ.cu", 0, [], [])
    assert err == nvrtc.nvrtcResult.NVRTC_SUCCESS
    opts = [b"--gpu-architecture=sm_100a"]
    err, = nvrtc.nvrtcCompileProgram(prog, len(opts), opts)
    assert err == nvrtc.nvrtcResult.NVRTC_SUCCESS
    err, size = nvrtc.nvrtcGetCUBINSize(prog)
    cubin = b" " * size
    err, = nvrtc.nvrtcGetCUBIN(prog, cubin)
    assert err == nvrtc.nvrtcResult.NVRTC_SUCCESS
    err, mod = driver.cuModuleLoadData(cubin)
    assert err == driver.CUresult.CUDA_SUCCESS
    err, fn = driver.cuModuleGetFunction(mod, b"k")
    assert err == driver.CUresult.CUDA_SUCCESS
    err, = driver.cuFuncSetAttribute(
        fn, driver.CUfunction_attribute.CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, 232448)
    assert err == driver.CUresult.CUDA_SUCCESS

    def blocks(threads, smem):
        err, n = driver.cuOccupancyMaxActiveBlocksPerMultiprocessor(fn, threads, smem)
        assert err == driver.CUresult.CUDA_SUCCESS
        return n
    return blocks


@pytest.mark.gpu
def test_b200_shmem_occupancy_vs_fig12():
    import torch
    props = torch.cuda.get_device_properties(0)
    if (props.major, props.minor) != (10, 0):
        pytest.skip("B200 (cc 10.0) only")
    blocks = _calculator()
    rows = []
    for threads in (128, 256, 512):
        for spb in (2048, 4096, 8192, 16384, 24576, 32768, 49152, 65536, 100352, 116736, 232448):
            cuda = blocks(threads, spb)
            paper = min(SMEM_SM // spb, MAX_BLOCKS)                      # Fig 12, no thread cap (A12)
            # the same with the 1 KB per-block reservation (reading A11) and
            # the thread limit the paper leaves out (A12)
            reserved = min(SMEM_SM // (spb + 1024), MAX_BLOCKS, THREADS_SM // threads)
            rows.append((threads, spb, paper, cuda, reserved))
            assert cuda == reserved, rows[-1]
            assert min(paper, THREADS_SM // threads) >= cuda, rows[-1]
    # the gap is real: e.g. 16 KB blocks (paper 14, hardware 13 per SM)
    assert any(min(p, THREADS_SM // t) > c for t, _, p, c, _ in rows)
