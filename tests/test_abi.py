"""The C-ABI library loads on a CPU-only machine and exports every symbol that
include/mg.h declares; the Python binding covers exactly those names; the
product package never imports the oracle; no CPU fallback exists."""
import ast
import os
import re
import subprocess

import pytest

from paper_conf_sc_antepara0jh24_b200 import mg

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "mg.h")


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:mg_status|void|const char\*)\s+(mg_\w+)\s*\(", src, flags=re.M)))


def test_header_declares_the_survey_boundary():
    names = declared_functions()
    for must in ("mg_setup", "mg_vcycle", "mg_solve", "mg_residual_norm", "mg_set_rhs", "mg_get_solution",
                 "mg_destroy", "mg_last_error", "mg_workspace_bytes", "mg_nccl_unique_id"):
        assert must in names


def test_library_exports_every_declared_symbol():
    lib = mg.lib()
    out = subprocess.run(["nm", "-D", "--defined-only", mg.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (mg_\w+)", out))
    for name in declared_functions():
        assert name in exported, name
        assert getattr(lib, name) is not None


def test_binding_covers_header_exactly():
    assert sorted(mg.header_symbols()) == declared_functions()


def test_library_is_sm100a_and_links_nccl():
    out = subprocess.run(["cuobjdump", "--list-elf", mg.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    deps = subprocess.run(["ldd", mg.LIB_PATH], capture_output=True, text=True).stdout
    assert "libnccl.so.2" in deps


def test_setup_without_gpu_fails_loudly():
    """No CPU fallback: on a machine without a CUDA device mg_setup errors."""
    import torch

    if torch.cuda.is_available():
        pytest.skip("GPU present")
    p = mg.params((32, 32, 32), num_levels=2)
    with pytest.raises(mg.MGError) as e:
        mg.mg_setup(p, 0, 1, None, 0, None, None, 0)
    assert e.value.status == -2  # MG_ERR_CUDA


def test_product_package_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_sc_antepara0jh24_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            path = os.path.join(dirpath, f)
            if f.endswith(".py"):
                tree = ast.parse(open(path).read())
                for node in ast.walk(tree):
                    if isinstance(node, ast.Import):
                        assert not any(a.name.split(".")[0] == "oracle" for a in node.names), path
                    if isinstance(node, ast.ImportFrom):
                        assert (node.module or "").split(".")[0] != "oracle", path
            if f.endswith((".cu", ".cpp", ".h")):
                assert "oracle" not in open(path).read().lower() or f == "kernels.cu", path


def test_workspace_bytes_scales_with_levels():
    a = mg.mg_workspace_bytes(mg.params((64, 64, 64), num_levels=1))
    b = mg.mg_workspace_bytes(mg.params((64, 64, 64), num_levels=4))
    assert b > a and a >= 4 * 64**3 * 8  # x, x' (ping-pong), b, r


def test_workspace_holds_ax_only_for_the_paper_kernel_set():
    """Ax (applyOp's output) exists only on levels that run the paper's kernel set (fusion 1); the
    host-upload staging fields are allocated on first use, outside the workspace."""
    n = 64
    fused = mg.mg_workspace_bytes(mg.params((n, n, n), num_levels=1))
    paper = mg.mg_workspace_bytes(mg.params((n, n, n), num_levels=1, fusion=[1] + [0] * 15))
    assert paper - fused >= n**3 * 8 and paper - fused <= n**3 * 8 + 4096 + 256  # + the zero brick, alignment
    assert fused < 5 * n**3 * 8


@pytest.mark.parametrize("n,L,launches", [(512, 6, 88), (256, 6, 99), (64, 4, 73)])
def test_vcycle_launch_count(n, L, launches):
    """Launches of one V-cycle (the bench's launches_per_step): at 512^3, L = 6 level 0
    runs 6 pencil passes + 1 interpolation + 6 passes (13), levels 1 and 2 a zero-folded single
    sweep, 5 passes and a restricting single sweep, then an interpolation and 6 passes (14 each),
    levels 3 and 4 24 single sweeps each (the first post-sweep with the interpolation fused), the
    bottom 1 resident launch: 90."""
    lay = mg.Layout(mg.params((n, n, n), num_levels=L))
    assert lay.vcycle_launches() == launches


@pytest.mark.parametrize("bad", [dict(smoother=3), dict(launch_pdl=3), dict(bottom_solver=2), dict(smoother=-1), dict(bottom_mode=5), dict(transport=7),
                                 dict(num_levels=2, pre=0)])
def test_invalid_parameters_are_rejected_without_a_gpu(bad):
    """Parameter validation (mg_workspace_bytes, the first call of a setup) rejects unknown
    smoothers, bottom modes, transports and pre = 0 with more than one level (the restriction
    reads the last pre-sweep's r) -- MG_ERR_INVALID_ARG with a message, no crash."""
    from paper_conf_sc_antepara0jh24_b200 import mg

    kw = dict(num_levels=3)
    kw.update(bad)
    with pytest.raises(mg.MGError) as e:
        mg.mg_workspace_bytes(mg.params((64, 64, 64), **kw))
    assert e.value.status == -1 and str(e.value)


@pytest.mark.parametrize("smoother", [0, 1, 2])
def test_smoother_variants_need_no_extra_workspace(smoother):
    from paper_conf_sc_antepara0jh24_b200 import mg

    base = mg.mg_workspace_bytes(mg.params((64, 64, 64), num_levels=3))
    assert mg.mg_workspace_bytes(mg.params((64, 64, 64), num_levels=3, smoother=smoother)) == base
