"""CPU-side checks of the C ABI (-m "not gpu"): libpf.so builds for sm_100a,
loads without a GPU, exports every function include/pf.h declares, and the
ctypes mirrors of the ABI structs match the C layout (sizes and offsets
measured by compiling a probe against include/pf.h with the host compiler).
No compute calls are made here."""
import ctypes as C
import os
import re
import subprocess
import tempfile

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "pf.h")


def declared_functions():
    src = open(HDR).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:const\s+)?\w+\**\s+\**(pf_\w+)\s*\(", src, flags=re.M)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_sc_0003hehshhkwnr19_b200 import build, pf
    build.build()
    return pf.load_library()


def test_header_declares_the_north_star_calls():
    f = declared_functions()
    for name in ("pf_create", "pf_set_params", "pf_init_fields", "pf_step", "pf_halo_exchange",
                 "pf_shift_window", "pf_download"):
        assert name in f


def test_library_exports_every_declared_symbol(lib):
    from paper_conf_sc_0003hehshhkwnr19_b200 import pf
    decl = declared_functions()
    assert sorted(pf.ABI_SYMBOLS) == decl
    for name in decl:
        assert hasattr(lib, name), name
    assert b"sm_100a" in lib.pf_version()


def test_library_is_sm100a_cubin():
    from paper_conf_sc_0003hehshhkwnr19_b200 import build
    so = build.build()
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", so], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_struct_layout_matches_c(lib):
    from paper_conf_sc_0003hehshhkwnr19_b200 import pf
    probe = r'''
#include <stdio.h>
#include <stddef.h>
#include "pf.h"
int main(void) {
  printf("%zu %zu %zu %zu\n", sizeof(pf_config), sizeof(pf_layout), sizeof(pf_params), sizeof(pf_state));
  printf("%zu %zu %zu %zu\n", offsetof(pf_config, stream), offsetof(pf_config, workspace),
         offsetof(pf_params, D), offsetof(pf_params, window_check));
  printf("%zu %zu\n", offsetof(pf_layout, pitch), offsetof(pf_layout, workspace_bytes));
  printf("%zu %zu\n", sizeof(pf_tuning), offsetof(pf_tuning, mu_ty));
  return 0;
}
'''
    with tempfile.TemporaryDirectory() as d:
        c = os.path.join(d, "probe.c")
        open(c, "w").write(probe)
        exe = os.path.join(d, "probe")
        subprocess.check_call(["gcc", "-std=c99", "-I", os.path.dirname(HDR), c, "-o", exe])
        vals = [int(v) for v in subprocess.check_output([exe], text=True).split()]
    got = [C.sizeof(pf.PFConfig), C.sizeof(pf.PFLayout), C.sizeof(pf.PFParams), C.sizeof(pf.PFState),
           pf.PFConfig.stream.offset, pf.PFConfig.workspace.offset, pf.PFParams.D.offset,
           pf.PFParams.window_check.offset, pf.PFLayout.pitch.offset, pf.PFLayout.workspace_bytes.offset,
           C.sizeof(pf.PFTuning), pf.PFTuning.mu_ty.offset]
    assert got == vals


def test_no_oracle_in_product_path():
    """The product package never imports or links the oracle (task rule 3)."""
    pkg = os.path.join(ROOT, "paper_conf_sc_0003hehshhkwnr19_b200")
    for dp, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                s = open(os.path.join(dp, f)).read()
                for pat in (r"^\s*(from|import)\s+oracle", r"#include\s+[<\"].*oracle", r"pf_oracle", r"oracle_\w+\("):
                    assert not re.search(pat, s, flags=re.M), (f, pat)


def test_specialised_kernels_compile_without_gpu(lib, tmp_path):
    """The run-time specialisation (NVRTC, sm_100a) builds for the C.4 and
    stress parameter sets and every liquid index, with no device present."""
    from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I
    from paper_conf_sc_0003hehshhkwnr19_b200 import pf
    cub = str(tmp_path / "k.cubin")
    assert pf.jit_compile_only(I.params_c4("ds"), n=48, cubin_path=cub) > 0
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", cub], capture_output=True, text=True).stdout
    assert "pf_jit_mu" in out and "DFMA" in out
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", cub + ".phi"], capture_output=True, text=True).stdout
    assert "pf_jit_phi" in out and "DFMA" in out
    assert pf.jit_compile_only(dict(I.params_stress(), liquid=1), n=17) > 0


def test_tuning_defaults_and_range_check(lib):
    """pf_tuning_default / pf_tuning_check (NEXT-2): the defaults are valid,
    values outside the documented ranges are rejected with a reason."""
    from paper_conf_sc_0003hehshhkwnr19_b200 import pf
    t = pf.tuning_default()
    assert set(t) == set(pf.TUNING_KNOBS)
    assert pf.tuning_check(t) == "ok"
    for bad in ({"phi_ty": 5}, {"mu_ty": 2}, {"mu_tx": 16, "mu_ty": 3}, {"mu_minb": 7}, {"phi_unroll": 0},
                {"mu_pfd": 1}, {"phi_minb": 8, "phi_ty": 16}, {"mu_rpf": 2}, {"mu_zc": 1000},
                {"mu_cly": 3}, {"mu_cly": 2, "mu_tx": 16, "mu_ty": 4}, {"mu_rot": 2}, {"mu_rpt": 3},
                {"mu_ty": 4}, {"mu_qreg": 1}, {"mu_cly": 2}, {"phi_rpt": 2, "phi_faces6": 0},
                {"phi_rpt": 2, "phi_xsh": 1}, {"mu_ty": 7, "mu_minb": 1}, {"mu_ty": 18, "mu_minb": 1},
                {"mu_rpt": 1, "mu_ty": 16, "mu_minb": 1}):
        msg = pf.tuning_check(dict(t, **bad))
        assert msg != "ok", bad
    # taller two-rows tiles are valid (one CTA per SM; measured slower)
    assert pf.tuning_check(dict(t, mu_ty=16, mu_minb=1)) == "ok"


@pytest.mark.parametrize("knobs", [
    {"phi_ty": 16, "phi_minb": 1, "phi_faces6": 0, "phi_unroll": 4, "phi_prefetch": 2, "phi_pfd": 3,
     "mu_ty": 8, "mu_tx": 16, "mu_minb": 4, "mu_rpf": 0, "mu_halo_l1": 0, "mu_fxreg": 0, "mu_prefetch": 0,
     "phi_xghost": 1, "mu_ldhint": 2, "mu_qreg": 1, "mu_rpt": 1},
    {"phi_ty": 8, "phi_minb": 2, "phi_zc": 32, "phi_prefetch": 0, "mu_ty": 3, "mu_minb": 5, "mu_zc": 24,
     "mu_pfd": 3, "mu_prefetch": 2, "mu_rpt": 1},
    {"mu_cly": 4, "mu_rot": 1, "mu_rpt": 1, "mu_ty": 4, "mu_minb": 3},
    {"mu_cly": 2, "mu_ty": 6, "mu_minb": 2, "mu_qreg": 1, "mu_fxreg": 0, "mu_hpipe": 1, "mu_rpt": 1},
    {"mu_rpt": 2, "mu_ty": 6, "mu_minb": 2, "mu_rpf": 0, "mu_prefetch": 2},
    {"phi_rpt": 2, "phi_ty": 16, "phi_minb": 1, "phi_unroll": 2, "phi_xghost": 1},
    # halo ring staged by cp.async (1), whole-tile staging (2), without the
    # register prefetch (falls back to 1), the concurrent slab schedule
    {"mu_hasync": 1, "mu_halo_l1": 0, "mu_zc": 7},
    {"mu_hasync": 2, "mu_ty": 6, "mu_minb": 3},
    {"mu_hasync": 2, "mu_rpf": 0},
    {"sched": 2, "slab": 2, "mu_hasync": 1},
])
def test_tuned_variants_compile_without_gpu(lib, knobs):
    """Extreme corners of the auto-tuning space (pf_autotune's knobs) still
    build with NVRTC for sm_100a."""
    from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I
    from paper_conf_sc_0003hehshhkwnr19_b200 import pf
    t = dict(pf.tuning_default(), **knobs)
    assert pf.tuning_check(t) == "ok"
    assert pf.jit_compile_only(I.params_c4("ds"), n=40, tuning=t) > 0


def test_p2_layout_and_params_struct():
    """P2 (NEXT-4) through the same ABI: 3 phase and 1 mu components per
    buffer; pf_params carries the anisotropy (aniso, aniso_delta, aniso_R)."""
    from paper_conf_sc_0003hehshhkwnr19_b200 import build, inputs as I, pf
    build.build()
    L1 = pf.query_layout((20, 24, 40))
    L2 = pf.query_layout((20, 24, 40), n_phases=3, n_mu=1)
    assert (L1.pitch, L1.plane, L1.field) == (L2.pitch, L2.plane, L2.field)
    assert L2.phi_bytes == 3 * L2.field * 8 + 256 and L2.mu_bytes == L2.field * 8 + 256
    assert L1.phi_bytes == 4 * L1.field * 8 + 256 and L1.mu_bytes == 2 * L1.field * 8 + 256
    p = pf.make_params(I.params_p2_stress())
    P = I.params_p2_stress()
    assert p.aniso == 1
    assert abs(p.aniso_R[0][2][1][0] - P["aniso_R"][0, 2, 1, 0]) == 0.0
    assert p.aniso_delta[1][2] == P["aniso_delta"][1, 2]
    assert p.A0[2][0][0] == P["A0"][2, 0, 0] and p.D[1][0][0] == P["D"][1, 0, 0]


@pytest.mark.parametrize("knobs", [{}, {"p2_phi": 1, "p2_mu": 1}, {"p2_phi": 2, "p2_mu": 2},
                                   {"p2_phi_ty": 4, "p2_phi_minb": 4, "p2_mu_ty": 8, "p2_mu_minb": 1, "p2_phi_pd": 0},
                                   {"p2_phi": 0, "p2_mu_hasync": 0}, {"p2_mu_ty": 4, "p2_mu_minb": 6, "p2_mu_hasync": 1}])
def test_p2_specialised_kernels_compile_without_gpu(lib, tmp_path, knobs):
    """The run-time specialised P2 sweeps (pf_p2_dev.cuh on compile-time
    parameters) build with NVRTC for every kernel choice; with the P2 set
    (isotropic unrotated solid-solid pair, one unrotated grain) the phi-sweep
    issues far fewer fp64 instructions than the generic stress-set build."""
    from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I
    from paper_conf_sc_0003hehshhkwnr19_b200 import pf
    t = dict(pf.tuning_default(), **knobs)
    assert pf.tuning_check(t) == "ok"
    cub = str(tmp_path / "p2.cubin")
    assert pf.jit_compile_only_p2(I.params_p2(), cubin_path=cub, tuning=t) > 0
    assert pf.jit_compile_only_p2(dict(I.params_p2_stress(), liquid=0), cubin_path=cub + "s", tuning=t) > 0

    def fp64(path):
        out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", path], capture_output=True, text=True).stdout
        assert "pf_p2_jit" in out
        return len(re.findall(r"\b(DFMA|DADD|DMUL)\b", out))
    if not knobs:
        assert fp64(cub + ".phi") < 0.8 * fp64(cub + "s.phi")
