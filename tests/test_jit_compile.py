"""The plan-specialised kernels (csrc/jit.cpp) are compiled at run time by NVRTC from the
library's own kernel.cu.  NVRTC needs no GPU, so this CPU test compiles that source exactly as
jit.cpp does (same headers, options and plan record) for an undirected, a labeled vertex-
induced and a directed plan, so a change that breaks the JIT compile fails here and not only
on the GPU box."""
import ctypes
import os

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CSRC = os.path.join(ROOT, "paper_conf_sc_weij22_b200", "csrc")
NVRTC = "/usr/local/cuda/lib64/libnvrtc.so"


def _plan_header(raw: bytes, k: int) -> str:
    return (f"#define STM_CPLAN_K {k}\n__device__ const StmPlanBytes kCPlan = {{{{"
            + ",".join(str(b) for b in raw) + "}};\n")


@pytest.mark.skipif(not os.path.exists(NVRTC), reason="no NVRTC")
@pytest.mark.parametrize("case", ["k5", "house_vi_labeled", "directed_cycle3"])
def test_specialised_kernel_compiles(case):
    from paper_conf_sc_weij22_b200 import stm
    import stmgen
    if case == "k5":
        p = stmgen.CATALOG["k5"]
        plan, variant = stm.Plan(p.k, p.edges), 2
    elif case == "house_vi_labeled":
        p = stmgen.CATALOG["house"]
        plan, variant = stm.Plan(p.k, p.edges, (0, 1, 2, 0, 1), vertex_induced=True), 1
    else:
        plan, variant = stm.Plan(3, [(0, 1), (1, 2), (2, 0)], directed=True), 2
    nv = ctypes.CDLL(NVRTC)
    src = open(os.path.join(CSRC, "kernel.cu")).read().encode()
    hdrs = {n: open(os.path.join(CSRC, n)).read() for n in ("kernel.h", "plan.h", "stm_nvrtc_prelude.h")}
    hdrs["stm_cplan.h"] = _plan_header(stm.stm_plan_raw(plan.handle), plan.k)
    names = list(hdrs)
    H = (ctypes.c_char_p * len(names))(*[hdrs[n].encode() for n in names])
    N = (ctypes.c_char_p * len(names))(*[n.encode() for n in names])
    prog = ctypes.c_void_p()
    assert nv.nvrtcCreateProgram(ctypes.byref(prog), src, b"kernel.cu", len(names), H, N) == 0
    opts = [b"--gpu-architecture=sm_100a", b"-std=c++17", b"-lineinfo", b"-DSTM_NVRTC=1", b"-DSTM_CPLAN=1",
            b'-DSTM_CPLAN_HEADER="stm_cplan.h"', f"-DSTM_JIT_VARIANT={variant}".encode()]
    O = (ctypes.c_char_p * len(opts))(*opts)
    rc = nv.nvrtcCompileProgram(prog, len(opts), O)
    n = ctypes.c_size_t()
    nv.nvrtcGetProgramLogSize(prog, ctypes.byref(n))
    log = ctypes.create_string_buffer(n.value)
    nv.nvrtcGetProgramLog(prog, log)
    assert rc == 0, log.value.decode()[:2000]
    size = ctypes.c_size_t()
    assert nv.nvrtcGetCUBINSize(prog, ctypes.byref(size)) == 0 and size.value > 0
    cubin = ctypes.create_string_buffer(size.value)
    assert nv.nvrtcGetCUBIN(prog, cubin) == 0
    name = b"stm_count_kernel_occ" if variant == 2 else b"stm_count_kernel"
    assert name in cubin.raw  # the extern "C" entry jit.cpp looks up
    nv.nvrtcDestroyProgram(ctypes.byref(prog))
