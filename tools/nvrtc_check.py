"""Compile a run-time GAS program the way gr_program_compile does (NVRTC, the
embedded device headers, every kernel name the drivers look up) WITHOUT a GPU,
to catch compile errors before a gpurun. Usage: python tools/nvrtc_check.py"""
import ctypes
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
from paper_conf_sc_senguptasas15_b200 import _build  # noqa: E402

nv = ctypes.CDLL("/usr/local/cuda/lib64/libnvrtc.so.12")


def compile_prog(src, name, arch="sm_100a"):
    names, srcs = [], []
    for n, path in _build.JIT_HEADERS:
        names.append(n.encode())
        srcs.append(open(path).read().encode())
    for n, text in _build.JIT_STANDINS.items():
        names.append(n.encode())
        srcs.append(text.replace("\\n", "\n").encode())
    P = "gr::" + name
    tu = ('#define GR_JIT 1\n#include "kernels_stream.cuh"\nnamespace gr {\n#line 1 "user_program"\n' + src +
          "\n}  // namespace gr\n")
    kernels = ["k_persistent", "k_init_values", "k_init_frontier", "k_init_edges", "k_s_init_scatter",
               "k_s_gather_apply", "k_s_activate", "k_gather_apply", "k_gather_apply_x", "k_scatter_activate"]
    exprs = [f"gr::{k}<{P}, {o}>" for k in kernels for o in ("unsigned int", "unsigned long long")]
    exprs.append(f"gr::k_prog_fill<{P}>")
    prog = ctypes.c_void_p()
    N = len(names)
    arr = ctypes.c_char_p * N
    rc = nv.nvrtcCreateProgram(ctypes.byref(prog), tu.encode(), b"gr_user_program.cu", N, arr(*srcs), arr(*names))
    assert rc == 0, rc
    for e in exprs:
        nv.nvrtcAddNameExpression(prog, e.encode())
    opts = [f"--gpu-architecture={arch}".encode(), b"-std=c++17", b"-default-device"]
    rc = nv.nvrtcCompileProgram(prog, len(opts), (ctypes.c_char_p * len(opts))(*opts))
    ls = ctypes.c_size_t()
    nv.nvrtcGetProgramLogSize(prog, ctypes.byref(ls))
    log = ctypes.create_string_buffer(ls.value + 1)
    nv.nvrtcGetProgramLog(prog, log)
    return rc, log.value.decode(errors="replace")


if __name__ == "__main__":
    from test_gpu_parity import JIT_SSSP, JIT_CC64  # noqa: E402
    from test_gpu_programs import JIT_HEAT  # noqa: E402

    for src, name in ((JIT_SSSP, "JitSSSP"), (JIT_CC64, "JitCC64"), (JIT_HEAT, "JitHeat")):
        rc, log = compile_prog(src, name)
        print(name, "rc", rc)
        if rc:
            print(log[-3000:])
            sys.exit(1)
