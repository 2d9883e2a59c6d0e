"""GPU parity: the CUDA path (through the C ABI) against the oracle.

Bars (BASELINE.json north_star):
  * integer outputs bit-exact: permuted CSR (row_ptr, col, value bits), stream
    tiles, row classes, hub chunks, partition bounds, H, inverse perm;
  * y within |y_gpu - y_ref| <= 1e-5 * sum_j |a_rj x_j| per row (TOL below);
  * y bitwise repeatable and independent of the row partition (world).
"""
import math

import numpy as np
import pytest

import synth
from oracle import cref, permute, plan as oplan, power, rabbit, spmv as ospmv

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
TOL = 1e-5


def _skip_no_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


@pytest.fixture(scope="module")
def dev():
    _skip_no_gpu()
    from paper_conf_ispass_balajicjk23_b200 import spmv  # noqa: F401  (fails loudly if missing)
    return torch.device("cuda:0")


def to_dev(A, dev, rp_dtype=torch.int64):
    return (torch.from_numpy(np.asarray(A.row_ptr)).to(dev, rp_dtype),
            torch.from_numpy(np.asarray(A.col)).to(dev),
            torch.from_numpy(np.asarray(A.val)).to(dev))


def mk_plan(A, perm, dev, **kw):
    from paper_conf_ispass_balajicjk23_b200 import spmv
    rp, c, v = to_dev(A, dev, kw.pop("rp_dtype", torch.int64))
    p = None if perm is None else torch.from_numpy(np.asarray(perm, np.int32)).to(dev)
    return spmv.Plan(rp, c, v, p, **kw)


class Mat:
    def __init__(self, n, row_ptr, col, val):
        self.n, self.row_ptr, self.col, self.val = n, np.asarray(row_ptr, np.int64), \
            np.asarray(col, np.int32), np.asarray(val, np.float32)

    @property
    def nnz(self):
        return int(self.row_ptr[-1])


def long_rows_matrix(seed=0):
    """Rows of every class: empty, short, medium, CTA, hub (> 16384), with
    duplicates and unsorted columns."""
    rng = np.random.default_rng(seed)
    n = 30000
    L = rng.integers(0, 20, n)
    L[rng.random(n) < 0.3] = 0
    special = {5: 40000, 17: 16385, 99: 16384, 1000: 9000, 1001: 2049, 1002: 2048, 2500: 700,
               2501: 33, 2502: 32, 3000: 3000, 3001: 5, 3002: 7, 3500: 1500, 3501: 3,
               29999: 70000}
    for r, l in special.items():
        L[r] = l
    rp = np.concatenate([[0], np.cumsum(L)])
    col = rng.integers(0, n, rp[-1]).astype(np.int32)
    col[rp[5]:rp[5] + 100] = 7                       # duplicates in a hub row
    val = rng.uniform(-1, 1, rp[-1]).astype(np.float32)
    return Mat(n, rp, col, val)


def _cases():
    yield "rmat12", lambda: synth.config(1, small=True).A
    yield "sbm16x1024", lambda: synth.config(2, small=True).A
    yield "stencil24", lambda: synth.config(4, small=True).A
    yield "kron14", lambda: synth.config(5, small=True).A
    yield "longrows", long_rows_matrix


CASES = list(_cases())


def _perms(A, which):
    if which == "identity":
        return None
    if which == "random":
        return rabbit.random_perm(A.n, 77)
    if which == "rabbitpp":
        from paper_conf_ispass_balajicjk23_b200 import spmv
        return spmv.reorder(A.row_ptr, A.col, "rabbitpp")[0]
    raise ValueError(which)


@pytest.mark.parametrize("name,make", CASES)
@pytest.mark.parametrize("which", ["identity", "random", "rabbitpp"])
def test_permute_and_bins_bitexact(dev, name, make, which):
    A = make()
    if which == "rabbitpp" and name == "longrows":
        which = "random"
    perm = _perms(A, which)
    P = mk_plan(A, perm, dev)
    pm = np.arange(A.n) if perm is None else np.asarray(perm, np.int64)
    Bp, Bc, Bv = permute.permute_csr(A.n, A.row_ptr, A.col, A.val, pm)
    rp, c, v = (t.cpu().numpy() for t in P.export_csr())
    assert np.array_equal(rp, Bp)
    assert np.array_equal(c, Bc)
    assert np.array_equal(v.view(np.int32), Bv.view(np.int32))
    bins = {k: t.cpu().numpy() for k, t in P.export_bins().items()}
    assert np.array_equal(bins["tiles"], oplan.tile_bounds(Bp))
    warp, cta, hub, cr, ci = oplan.row_classes(Bp)
    assert np.array_equal(bins["mid_rows"], oplan.mid_rows(Bp))
    assert np.array_equal(bins["warp_rows"], warp)
    assert np.array_equal(bins["cta_rows"], cta)
    assert np.array_equal(bins["hub_rows"], hub)
    assert np.array_equal(bins["chunk_row"], cr) and np.array_equal(bins["chunk_idx"], ci)
    info = P.info()
    assert info["hot_prefix"] == oplan.hot_prefix(A.n, Bc)
    assert np.array_equal(P.export_inverse().cpu().numpy(), permute.inverse(pm))
    P.close()


def _check_y(y, ref, absrow, what=""):
    err = np.abs(y.astype(np.float64) - ref.astype(np.float64))
    bad = err > TOL * absrow + 1e-37
    assert not bad.any(), f"{what}: {bad.sum()} rows out of tolerance, worst {err[bad].max()}"


@pytest.mark.parametrize("name,make", CASES)
def test_exec_matches_oracle(dev, name, make):
    A = make()
    perm = rabbit.random_perm(A.n, 5)
    P = mk_plan(A, perm, dev)
    x = synth.vector(A.n, 99)
    Bp, Bc, Bv = permute.permute_csr(A.n, A.row_ptr, A.col, A.val, perm)
    xB = permute.permute_vec(x, perm)
    xB_dev = P.permute_vec(torch.from_numpy(x).to(dev))
    assert np.array_equal(xB_dev.cpu().numpy(), xB)
    y = P.exec(xB_dev).cpu().numpy()
    ref = ospmv.spmv(Bp, Bc, Bv, xB)
    _check_y(y, ref, ospmv.abs_rowsum(Bp, Bc, Bv, xB), name)
    # empty rows give exactly +-0
    L = np.diff(Bp)
    assert np.all(y[L == 0] == 0)
    # bitwise repeatable
    y2 = P.exec(xB_dev).cpu().numpy()
    assert np.array_equal(y.view(np.int32), y2.view(np.int32))
    # P^T y_B == A x  (inverse relabel on the device)
    yA = P.permute_vec(torch.from_numpy(y).to(dev), inverse=True).cpu().numpy()
    _check_y(yA, ospmv.spmv(A.row_ptr, A.col, A.val, x), ospmv.abs_rowsum(A.row_ptr, A.col, A.val, x))
    P.close()


@pytest.mark.parametrize("name,make", [c for c in CASES if c[0] in ("rmat12", "longrows", "kron14")])
@pytest.mark.parametrize("world", [2, 3, 4])
@pytest.mark.parametrize("layout", ["global", "padded"])
def test_partitioned_equals_single_bitwise(dev, name, make, world, layout):
    A = make()
    perm = rabbit.random_perm(A.n, 11)
    P1 = mk_plan(A, perm, dev)
    x = torch.from_numpy(synth.vector(A.n, 3)).to(dev)
    xB = P1.permute_vec(x)
    y1 = P1.exec(xB).cpu().numpy()
    Bp, _, _ = permute.permute_csr(A.n, A.row_ptr, A.col, A.val, perm)
    bounds = oplan.partition(Bp, world)
    parts = []
    for r in range(world):
        from paper_conf_ispass_balajicjk23_b200 import spmv
        Pr = mk_plan(A, perm, dev, world=world, rank=r,
                     x_layout=spmv.XLAYOUT_PADDED if layout == "padded" else spmv.XLAYOUT_GLOBAL)
        assert Pr.export_partition() == bounds.tolist()
        info = Pr.info()
        assert (info["row_begin"], info["row_end"]) == (bounds[r], bounds[r + 1])
        xpad = Pr.pad_vec(xB, to_padded=True)
        if layout == "padded":
            assert xpad.numel() == info["x_len"] == world * info["x_stride"]
            assert info["y_offset"] == r * info["x_stride"]
        else:  # global layout: x_B itself, this rank's y slice at row_begin
            assert xpad.numel() == info["x_len"] == A.n
            assert info["y_offset"] == bounds[r]
        back = Pr.pad_vec(xpad, to_padded=False)
        assert torch.equal(back, xB)
        parts.append(Pr.exec(xpad).cpu().numpy())
        Pr.close()
    yc = np.concatenate(parts)
    assert np.array_equal(yc.view(np.int32), y1.view(np.int32))
    P1.close()


def test_int32_and_int64_row_ptr_agree(dev):
    A = synth.config(1, small=True).A
    perm = rabbit.random_perm(A.n, 2)
    x = torch.from_numpy(synth.vector(A.n, 1)).to(dev)
    ys = []
    for dt in (torch.int32, torch.int64):
        P = mk_plan(A, perm, dev, rp_dtype=dt)
        ys.append(P.exec(P.permute_vec(x)).cpu().numpy())
        P.close()
    assert np.array_equal(ys[0].view(np.int32), ys[1].view(np.int32))


def test_errors(dev):
    from paper_conf_ispass_balajicjk23_b200 import spmv
    A = synth.rmat(8, 4, 1)
    bad = np.arange(A.n, dtype=np.int32)
    bad[3] = 4
    with pytest.raises(spmv.SpmvError) as e:
        mk_plan(A, bad, dev)
    assert e.value.status == 2  # EPERM
    Abad = Mat(A.n, A.row_ptr, np.where(A.col == 0, A.n, A.col), A.val)
    with pytest.raises(spmv.SpmvError) as e:
        mk_plan(Abad, None, dev)
    assert e.value.status == 1
    P = mk_plan(A, None, dev, permute=False)
    with pytest.raises(spmv.SpmvError) as e:
        P.exec(torch.zeros(A.n, device=dev))
    assert e.value.status == 7  # ESTATE
    P.close()


def test_degenerate_shapes(dev):
    for A in (Mat(1, [0, 0], [], []), Mat(5, [0] * 6, [], []),
              Mat(3, [0, 1, 1, 2], [2, 0], [2.5, -1.0]),
              Mat(2, [0, 70000, 70000], np.zeros(70000), np.ones(70000))):
        P = mk_plan(A, None, dev)
        x = np.arange(1, A.n + 1, dtype=np.float32)
        y = P.exec(torch.from_numpy(x).to(dev)).cpu().numpy()
        ref = ospmv.spmv(A.row_ptr, A.col, A.val, x)
        _check_y(y, ref, ospmv.abs_rowsum(A.row_ptr, A.col, A.val, x))
        P.close()


def test_iterate_regular_fixed_point(dev):
    # periodic 27-point stencil, unit values: lambda = 27, x0 = 1/sqrt(N) fixed
    A = synth.stencil27(12, periodic=True, relabel=True, seed_scr=5, valmode=synth.VAL_ONES)
    perm, _ = __import__("paper_conf_ispass_balajicjk23_b200").spmv.reorder(A.row_ptr, A.col, "rabbitpp")
    P = mk_plan(A, perm, dev)
    x0 = np.full(A.n, np.float32(1 / math.sqrt(A.n)))
    x = torch.from_numpy(x0).to(dev)
    lam = P.iterate(x, 10)
    assert math.isclose(lam, 27.0, rel_tol=1e-5)
    assert np.allclose(x.cpu().numpy(), x0, rtol=1e-5)
    P.close()


def test_iterate_matches_oracle_recurrence(dev):
    """20 power-iteration steps (reading c22) against the oracle recurrence.

    B >= 0 (Kronecker, values in (0, 1]) and x0 = |x| >= 0, so every iterate is
    nonnegative and a step's per-row error bound 1e-5 * sum_j |a x_j|
    (north_star) is a relative error of that row.  Through a nonnegative SpMV a
    componentwise relative error e of x gives at most e in every row of y (a
    weighted mean), the normalisation by s = ||y|| multiplies x by one common
    factor that the next step's s divides out again, and x = fp32(u / s) adds
    one rounding.  So the direction of x_t is within t * (1e-5 + 2^-23)
    componentwise, the final common factor within as much again: the bound
    below is 2 * iters * (1e-5 + 2^-23) * |x_ref| per entry, and lambda = s_t
    within 1e-5 relative (the last step's norm)."""
    w = synth.config(5, small=True)          # Kronecker, positive values
    A = w.A
    perm, _ = __import__("paper_conf_ispass_balajicjk23_b200").spmv.reorder(A.row_ptr, A.col, "rabbitpp")
    P = mk_plan(A, perm, dev)
    Bp, Bc, Bv = permute.permute_csr(A.n, A.row_ptr, A.col, A.val, perm)
    assert (np.asarray(Bv) > 0).all()
    x0 = np.abs(permute.permute_vec(w.x, perm)).astype(np.float32)
    x = torch.from_numpy(x0.copy()).to(dev)
    iters = 20
    lam = P.iterate(x, iters)
    xr, lr = power.power_iteration(Bp, Bc, Bv, x0, iters)
    assert abs(lam - lr) <= 1e-5 * lr
    bound = 2 * iters * (TOL + 2.0**-23)
    xg = x.cpu().numpy().astype(np.float64)
    assert np.all(np.abs(xg - xr) <= bound * np.abs(xr) + 1e-37)
    # step-wise parity: one scaled step from the GPU's own x
    xt = x.cpu().numpy()
    y = torch.empty(A.n, device=dev)
    ss = torch.zeros(1, dtype=torch.float64, device=dev)
    P.exec_scaled(x, y, None, ss)
    yr, sr = power.power_step(Bp, Bc, Bv, xt)
    _check_y(y.cpu().numpy(), yr, ospmv.abs_rowsum(Bp, Bc, Bv, xt))
    assert abs(math.sqrt(ss.item()) - sr) <= 1e-5 * sr
    P.close()


def _full_size_check(dev, cfg, ordering, nsample=2000, parallel=False):
    """BASELINE config `cfg` at full size, in the launch configuration bench.py
    times: sampled rows' integer structure against the oracle's own
    relabelling, sampled y against the exact fsum oracle, every row against
    the compensated C oracle on A itself, relabelled (y_B = P (A x))."""
    from paper_conf_ispass_balajicjk23_b200 import spmv
    w = synth.config(cfg)
    A = w.A
    if ordering == "original":
        perm = np.arange(A.n, dtype=np.int32)
    else:
        perm, _ = spmv.reorder(A.row_ptr, A.col, ordering, parallel=parallel)
    rp_dtype = torch.int32 if A.nnz < 2**31 else torch.int64
    P = mk_plan(A, perm, dev, rp_dtype=rp_dtype)
    xB = P.permute_vec(torch.from_numpy(w.x).to(dev))
    y = P.exec(xB).cpu().numpy()
    rp, c, v = (t.cpu().numpy() for t in P.export_csr())
    inv = permute.inverse(perm)
    rng = np.random.default_rng(cfg)
    rows = np.sort(rng.choice(A.n, min(nsample, A.n), replace=False))
    # the longest rows too (hub / CTA classes)
    L = np.diff(rp)
    rows = np.union1d(rows, np.argsort(L)[-20:])
    oracle_rows = permute.permute_rows(A.row_ptr, A.col, A.val, perm, inv, rows)
    for r, (cc, vv) in zip(rows, oracle_rows):
        assert np.array_equal(c[rp[r]:rp[r + 1]], cc)
        assert np.array_equal(v[rp[r]:rp[r + 1]].view(np.int32), vv.view(np.int32))
    xBh = permute.permute_vec(w.x, perm)
    ys = np.array([ospmv.spmv_rows([0, len(cc)], cc, vv, xBh, [0])[0] for cc, vv in oracle_rows])
    ab = np.array([np.abs(vv.astype(np.float64) * xBh[cc].astype(np.float64)).sum()
                   for cc, vv in oracle_rows])
    _check_y(y[rows], ys, ab, "sampled")
    assert np.all(y[L == 0] == 0)
    yA, absA = cref.spmv_neumaier(A.row_ptr, A.col, A.val, w.x)
    _check_y(y, permute.permute_vec(yA, perm), permute.permute_vec(absA, perm), "all rows")
    P.close()


def test_bench_config_full_size(dev):
    """BASELINE configs[1] (SBM 4M/64M, RABBIT++): the bench.py workload."""
    _full_size_check(dev, 2, "rabbitpp")


def test_rmat16_full_size(dev):
    """BASELINE configs[0] (RMAT scale 16) at full size, RABBIT++ order: every
    row against the exact fsum oracle as well."""
    _full_size_check(dev, 1, "rabbitpp", nsample=65536)


def test_rmat26_full_size(dev):
    """BASELINE configs[2] (RMAT scale 26, 67M rows, 1.06 B nnz, x = 268 MB >
    L2) at full size in its generated (ORIGINAL) order: hub rows (merge-path
    chunks + fp64 fixup), CTA rows, MID rows and lane rows at scale."""
    _full_size_check(dev, 3, "original")


def test_stencil464_full_size(dev):
    """BASELINE configs[3] (27-point stencil 464^3, 99.9 M rows, 2.69 G nnz) at
    full size as generated (random labels): the int64 row-pointer path
    (NZ >= 2^31), lane rows with shared 8-entry chunks, x = 400 MB > L2."""
    _full_size_check(dev, 4, "original", nsample=1000)


@pytest.mark.parametrize("name,make", CASES)
def test_smem_window_and_l2_options_bitwise(dev, name, make):
    """The x window, L2 policies and an unaligned x (window disabled) change
    where x is read from, never y."""
    from paper_conf_ispass_balajicjk23_b200 import spmv
    A = make()
    perm, _ = spmv.reorder(A.row_ptr, A.col, "rabbit")
    x = torch.from_numpy(synth.vector(A.n, 8)).to(dev)
    ys = []
    for kw in ({}, {"smem_window": False}, {"evict_first": False, "l2_window": False},
               {"variant": 1}, {"variant": 1, "smem_window": False}):
        P = mk_plan(A, perm, dev, **kw)
        xB = P.permute_vec(x)
        ys.append(P.exec(xB).cpu().numpy())
        buf = torch.zeros(A.n + 1, device=dev)
        buf[1:] = xB                      # 4-byte offset: not 16-byte aligned
        ys.append(P.exec(buf[1:]).cpu().numpy())
        P.close()
    for y in ys[1:]:
        assert np.array_equal(y.view(np.int32), ys[0].view(np.int32))


def test_exec_graph_capture_and_concurrency(dev):
    """exec forks the row-class kernels onto the plan's streams and joins them
    back: eager, CUDA-graph-captured and serial (SPMV_CONCURRENT=0) runs agree
    bitwise on a matrix with every row class."""
    import os
    A = long_rows_matrix(3)
    perm = rabbit.random_perm(A.n, 9)
    x = torch.from_numpy(synth.vector(A.n, 4)).to(dev)
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        P = mk_plan(A, perm, dev)
        xB = P.permute_vec(x)
        y0 = P.exec(xB)
        y1 = torch.full_like(y0, float("nan"))
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            P.exec(xB, y1)
        g.replay()
        torch.cuda.synchronize()
    assert torch.equal(y0.view(torch.int32), y1.view(torch.int32))
    P.close()
    os.environ["SPMV_CONCURRENT"] = "0"
    try:
        P = mk_plan(A, perm, dev)
        y2 = P.exec(P.permute_vec(x))
        torch.cuda.synchronize()
    finally:
        del os.environ["SPMV_CONCURRENT"]
    assert torch.equal(y0.view(torch.int32), y2.view(torch.int32))
    P.close()


def test_hot_x_option_removed(dev):
    """opts.hot_x > 0 (the removed hot-column set) is refused, not ignored."""
    from paper_conf_ispass_balajicjk23_b200 import spmv
    A = synth.config(1, small=True).A
    with pytest.raises(spmv.SpmvError):
        mk_plan(A, None, dev, hot_x=1)


@pytest.mark.parametrize("name,make", [c for c in CASES if c[0] != "longrows"])
def test_rabbitpp_gpu_postpass_bitexact(dev, name, make):
    """spmv_rabbitpp_gpu from the host RABBIT order and top-level
    communities equals the host RABBIT++ (and hence the oracle's, test_abi)."""
    from paper_conf_ispass_balajicjk23_b200 import spmv
    A = make()
    pr, _ = spmv.reorder(A.row_ptr, A.col, "rabbit")
    comm = spmv.reorder_last_comm(A.n)
    ppp, _ = spmv.reorder(A.row_ptr, A.col, "rabbitpp")
    out = spmv.rabbitpp_gpu(torch.from_numpy(A.row_ptr).to(dev), torch.from_numpy(A.col).to(dev),
                            torch.from_numpy(pr).to(dev), torch.from_numpy(comm).to(dev))
    assert np.array_equal(out.cpu().numpy(), ppp)
    out32 = spmv.rabbitpp_gpu(torch.from_numpy(A.row_ptr).to(dev, torch.int32),
                              torch.from_numpy(A.col).to(dev), torch.from_numpy(pr).to(dev),
                              torch.from_numpy(comm).to(dev))
    assert np.array_equal(out32.cpu().numpy(), ppp)


def test_rabbitpp_gpu_rejects_malformed_input(dev):
    """spmv_rabbitpp_gpu validates before indexing with its inputs: a perm
    that is not a bijection (EPERM), a community id or column out of range
    (EINVAL) are refused, never used as addresses."""
    from paper_conf_ispass_balajicjk23_b200 import spmv
    A = synth.config(1, small=True).A
    pr, _ = spmv.reorder(A.row_ptr, A.col, "rabbit")
    comm = spmv.reorder_last_comm(A.n)
    rp = torch.from_numpy(A.row_ptr).to(dev)
    col = torch.from_numpy(A.col).to(dev)
    bad_perm = pr.copy()
    bad_perm[0] = bad_perm[1]
    with pytest.raises(spmv.SpmvError) as e:
        spmv.rabbitpp_gpu(rp, col, torch.from_numpy(bad_perm).to(dev), torch.from_numpy(comm).to(dev))
    assert e.value.status == 2
    bad_comm = comm.copy()
    bad_comm[3] = A.n + 7
    with pytest.raises(spmv.SpmvError) as e:
        spmv.rabbitpp_gpu(rp, col, torch.from_numpy(pr).to(dev), torch.from_numpy(bad_comm).to(dev))
    assert e.value.status == 1
    bad_col = A.col.copy()
    bad_col[5] = -3
    with pytest.raises(spmv.SpmvError) as e:
        spmv.rabbitpp_gpu(rp, torch.from_numpy(bad_col).to(dev), torch.from_numpy(pr).to(dev),
                          torch.from_numpy(comm).to(dev))
    assert e.value.status == 1


def test_rmat26_rabbitpp_full_size(dev):
    """BASELINE configs[2] (RMAT-26) at full size in RABBIT++ order (concurrent
    RABBIT merges + the RABBIT++ post-pass): the hub-prefix persisting window,
    the stream cache policy and every row class at scale, sampled rows' CSR
    bit-exact and y within the tolerance, every row against the compensated C
    oracle."""
    _full_size_check(dev, 3, "rabbitpp", parallel=True)


@pytest.mark.parametrize("name,make", [c for c in CASES if c[0] in ("rmat12", "kron14", "stencil24")])
def test_small_plan_single_launch_bitwise(dev, name, make, monkeypatch):
    """Small plans (no hub rows, <= 2^24 entries) run every row class in one
    k_small launch: y and the scaled step's sum of y^2 bitwise equal to the
    separate per-class kernels, one launch (+2 for the norm) instead of up to
    three plus fork / join."""
    from paper_conf_ispass_balajicjk23_b200 import spmv
    A = make()
    perm = spmv.reorder(A.row_ptr, A.col, "rabbitpp")[0]
    P = mk_plan(A, perm, dev)
    i = P.info()
    xB = P.permute_vec(torch.from_numpy(synth.vector(A.n, 6)).to(dev))
    out = {}
    for mode in ("0", "1"):
        monkeypatch.setenv("SPMV_SMALL", mode)
        y = P.exec(xB)
        z = torch.empty_like(y)
        ss = torch.zeros(1, dtype=torch.float64, device=dev)
        P.exec_scaled(xB, z, None, ss)
        out[mode] = (y.clone(), z.clone(), ss.clone(), P.info()["exec_launches"])
    assert torch.equal(out["0"][0].view(torch.int32), out["1"][0].view(torch.int32))
    assert torch.equal(out["0"][1].view(torch.int32), out["1"][1].view(torch.int32))
    assert torch.equal(out["0"][2], out["1"][2])
    if i["n_mid_rows"] or i["n_cta_rows"]:
        assert out["1"][3] == 1
    monkeypatch.delenv("SPMV_SMALL")
    P.close()


@pytest.mark.parametrize("name,make", [c for c in CASES if c[0] in ("kron14", "stencil24", "sbm16x1024")])
def test_hot_prefix_window_gate(dev, name, make):
    """H and the entries it covers are exact (oracle plan.hot_prefix); exec
    pins x_B[0:H) in L2 only when those columns are read >= 2x as often as the
    average column (power-law hub groups yes, a stencil's near-average "hubs"
    no), at most half the L2."""
    from paper_conf_ispass_balajicjk23_b200 import spmv
    A = make()
    perm = spmv.reorder(A.row_ptr, A.col, "rabbitpp")[0]
    Bp, Bc, _ = permute.permute_csr(A.n, A.row_ptr, A.col, A.val, perm)
    H = oplan.hot_prefix(A.n, Bc)
    hot_nnz = int((Bc < H).sum())
    P = mk_plan(A, perm, dev)
    i = P.info()
    assert i["hot_prefix"] == H and i["hot_prefix_nnz"] == hot_nnz
    s = torch.cuda.Stream(device=dev)
    xB = torch.zeros(A.n, device=dev)
    P.exec(xB, stream=s)
    torch.cuda.synchronize()
    pays = H > 0 and hot_nnz * A.n >= 2 * A.nnz * H
    win = P.info()["l2_window_bytes"]
    assert (win > 0) == pays, (name, H, hot_nnz, win)
    l2 = torch.cuda.get_device_properties(dev).L2_cache_size
    assert win <= l2 // 2
    P.close()
