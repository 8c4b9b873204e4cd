"""NEXT-3: the tcgen05 combination kernel B = X*W (mps_xw_bf16) against fp64."""
import numpy as np
import pytest
import torch

import oracle as O

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_ispass_shangndk23_b200 as M


def _pad(a, ld):
    out = torch.zeros((a.shape[0], ld), dtype=a.dtype, device=a.device)
    out[:, : a.shape[1]] = a
    return out[:, : a.shape[1]]


@pytest.mark.parametrize("N", [16, 32, 48, 64, 128, 256])
@pytest.mark.parametrize("F", [16, 64, 72, 128])
def test_xw_exact_small_integers(N, F):
    # |sum| <= F <= 128 < 256: exact in fp32 accumulation AND in the bf16 output
    g = torch.Generator(device="cpu").manual_seed(N * 1000 + F)
    n = 1000 + 77                                   # ragged last tile
    X = torch.randint(-1, 2, (n, F), generator=g).to(torch.bfloat16).cuda()
    W = torch.randint(-1, 2, (F, N), generator=g).to(torch.bfloat16).cuda()
    B = M.xw_bf16(X, W.t().contiguous())
    ref = torch.from_numpy(O.xw_f64(X.float().cpu().numpy(), W.float().cpu().numpy()))
    assert torch.equal(B.double().cpu(), ref)


@pytest.mark.parametrize("n,F,N", [(5000, 602, 64), (2000, 100, 256), (129, 1433, 16), (40000, 128, 128)])
def test_xw_random_within_bf16_rounding(n, F, N):
    g = torch.Generator(device="cpu").manual_seed(n + F + N)
    ldx = (F + 7) // 8 * 8                          # TMA needs 16-B row strides
    X = _pad(torch.randn(n, F, generator=g).to(torch.bfloat16).cuda(), ldx)
    W = (torch.randn(F, N, generator=g) / F ** 0.5).to(torch.bfloat16)
    Wt = _pad(W.t().contiguous().cuda(), ldx)
    B = M.xw_bf16(X, Wt)
    Xd, Wd = X.double().cpu(), W.double()
    ref = torch.from_numpy(O.xw_f64(Xd.numpy(), Wd.numpy()))
    bound = torch.from_numpy(O.xw_f64(Xd.abs().numpy(), Wd.abs().numpy()))
    err = (B.double().cpu() - ref).abs()
    # bf16 output rounding (unit roundoff 2^-8) + fp32 accumulation of F products
    assert torch.all(err <= 2.0 ** -8 * ref.abs() + 1e-5 * bound + 1e-30)


def test_xw_unsupported_shapes_report_errors():
    X = torch.zeros((10, 64), dtype=torch.bfloat16, device="cuda")
    with pytest.raises(M.MpsError):
        M.xw_bf16(X, torch.zeros((20, 64), dtype=torch.bfloat16, device="cuda"))   # N % 16
    with pytest.raises(M.MpsError):
        M.xw_bf16(X, torch.zeros((272, 64), dtype=torch.bfloat16, device="cuda"))  # N > 256


def test_xw_unaligned_feature_width_is_padded():
    """F = 1433 (Cora's feature width): rows are not 16-B multiples; the binding pads."""
    g = torch.Generator(device="cpu").manual_seed(3)
    X = torch.randint(-1, 2, (500, 1433), generator=g).to(torch.bfloat16)
    W = torch.randint(-1, 2, (1433, 16), generator=g).to(torch.bfloat16)
    B = M.xw_bf16(X.cuda(), W.t().contiguous().cuda())
    ref = torch.from_numpy(O.xw_f64(X.float().numpy(), W.float().numpy()))
    # |sum| <= 1433: bf16 rounds, compare within one bf16 ulp of the exact integer
    assert torch.all((B.double().cpu() - ref).abs() <= ref.abs() * 2.0 ** -8)


def test_xw_streamed_w_when_w_does_not_fit():
    """Reddit K=256's combination (F = 602, N = 256: W = 308 KB > shared memory): the
    persistent kernel streams W chunks through the ring with X.  Within bf16 rounding of
    the fp64 oracle O9."""
    g = torch.Generator(device="cpu").manual_seed(602)
    n, F, N = 4097, 602, 256
    ldx = (F + 7) // 8 * 8
    X = _pad(torch.randn(n, F, generator=g).to(torch.bfloat16).cuda(), ldx)
    W = (torch.randn(F, N, generator=g) / F ** 0.5).to(torch.bfloat16)
    Wt = _pad(W.t().contiguous().cuda(), ldx)
    B = M.xw_bf16(X, Wt)
    Xd, Wd = X.double().cpu(), W.double()
    ref = torch.from_numpy(O.xw_f64(Xd.numpy(), Wd.numpy()))
    bound = torch.from_numpy(O.xw_f64(Xd.abs().numpy(), Wd.abs().numpy()))
    err = (B.double().cpu() - ref).abs()
    assert torch.all(err <= 2.0 ** -8 * ref.abs() + 1e-5 * bound + 1e-30)


def test_xw_streamed_w_forced_exact():
    """MPS_XW_WSTREAM=1 (W streamed even where it fits): the small-integer shapes stay
    bit-exact (the knob is read once per process: run in a subprocess)."""
    import os, subprocess, sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, MPS_XW_WSTREAM="1")
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-p", "no:cacheprovider",
                        os.path.join(root, "tests", "test_gpu_xw.py"), "-k",
                        "exact_small_integers"], env=env, capture_output=True, text=True,
                       timeout=600, cwd=root)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]


def test_xw_strided_output_keeps_padding():
    """The TMA-store epilogue writes B through a tensor map of the output's own row stride:
    a strided `out` (ldb > N) gets exactly its N columns, the padding keeps its sentinel,
    rows past a ragged last tile are not written (N = 64: whole 32-column chunks)."""
    g = torch.Generator(device="cpu").manual_seed(5)
    n, F, N, ldb = 1000 + 33, 64, 64, 96
    X = torch.randint(-1, 2, (n, F), generator=g).to(torch.bfloat16).cuda()
    W = torch.randint(-1, 2, (F, N), generator=g).to(torch.bfloat16).cuda()
    full = torch.full((n + 5, ldb), 7.0, dtype=torch.bfloat16, device="cuda")
    out = full[:n, :N]
    M.xw_bf16(X, W.t().contiguous(), out=out)
    ref = torch.from_numpy(O.xw_f64(X.float().cpu().numpy(), W.float().cpu().numpy()))
    assert torch.equal(out.double().cpu(), ref)
    assert torch.all(full[:, N:] == 7.0) and torch.all(full[n:] == 7.0)


@pytest.mark.parametrize("env", [{"MPS_XW_TMA_STORE": "0"}, {"MPS_XW_SPLIT": "2"},
                                 {"MPS_XW_STAGES": "8"}])
def test_xw_epilogue_variants_exact(env):
    """The per-lane store epilogue (MPS_XW_TMA_STORE=0), column slices on consecutive CTAs
    (MPS_XW_SPLIT=2: TMA stores at a column offset) and the full-depth ring for N >= F
    (MPS_XW_STAGES=8): the small-integer shapes stay bit-exact against O9 (the knobs are
    read once per process: run in a subprocess)."""
    import os, subprocess, sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-p", "no:cacheprovider",
                        os.path.join(root, "tests", "test_gpu_xw.py"), "-k",
                        "exact_small_integers or strided_output"], env=dict(os.environ, **env),
                       capture_output=True, text=True, timeout=900, cwd=root)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
