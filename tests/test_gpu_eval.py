"""GPU parity: batched evaluation kernels vs the oracle, element by element (bit-exact int64)."""
import json
import os

import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def lib():
    import torch

    assert torch.cuda.is_available()
    import paper_conf_ipps_awasthillw16_b200 as m

    return m


def _dev(x):
    import torch

    return torch.from_numpy(np.ascontiguousarray(x)).cuda()


def _gpu_eval(lib, inst, perms, problem="cdd", d=None):
    ins = lib.Instance(inst.P, inst.alpha, inst.beta, inst.d if d is None else d, inst.M, inst.gamma)
    fn = lib.cdd_eval_batch if problem == "cdd" else lib.ucddcp_eval_batch
    out = fn(ins, _dev(perms)).cpu().numpy()
    lib.cdd_check(ins)
    ins.destroy()
    return out


def _oracle(inst, perms, problem="cdd", d=None):
    pr = oracle.Problem.from_instance(inst, d=d)
    return oracle.eval_batch_threaded(pr, perms, oracle.CDD if problem == "cdd" else oracle.UCDDCP)


def test_table1(lib):
    t = gen.table1()
    perms = gen.random_perms(1, 5, 0)
    perms[0, :5] = np.arange(5)
    assert _gpu_eval(lib, t, perms)[0] == 81
    assert _gpu_eval(lib, t, perms, "ucddcp", d=22)[0] == 77


def test_config1_all_10_factorial(lib):
    # BASELINE config 1: CDD n=10, h=0.4, seed 1 -- every one of the 10! sequences
    gold = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "config1.json")))
    inst = gen.cdd_instance(10, 1, 0.4)
    perms = gen.all_perms(10)
    z = _gpu_eval(lib, inst, perms)
    ref = _oracle(inst, perms)
    assert np.array_equal(z, ref)
    assert int(z.min()) == gold["optimum"] and int(z.sum()) == gold["z_sum_over_all"]


@pytest.mark.parametrize("n", [1, 2, 3, 5, 7, 8, 9, 15, 16, 17, 31, 32, 33, 63, 64, 65, 100, 127,
                               128, 129, 200, 255, 256, 257, 333, 500, 511, 512, 513, 777, 999,
                               1000, 1023, 1024])
def test_random_instances_all_templates(lib, n):
    rng = np.random.default_rng(n)
    for h in (0.0, 0.2, 0.4, 0.6, 0.8, 1.0, 1.7):
        inst = gen.cdd_instance(n, 1 + n % 7, 0.2)
        d = int(h * inst.sum_p)
        B = 700 if n <= 256 else 150
        perms = gen.random_perms(B, n, int(rng.integers(1 << 30)))
        assert np.array_equal(_gpu_eval(lib, inst, perms, d=d), _oracle(inst, perms, d=d)), (n, h)


@pytest.mark.parametrize("n", [1, 4, 10, 17, 50, 100, 129, 200, 300, 500, 640, 1000, 1024])
def test_ucddcp_random(lib, n):
    inst = gen.ucddcp_instance(n, 2 + n % 5)
    B = 600 if n <= 256 else 120
    perms = gen.random_perms(B, n, 77 + n)
    for extra in (0, 13):
        d = inst.sum_p + extra
        assert np.array_equal(_gpu_eval(lib, inst, perms, "ucddcp", d=d),
                              _oracle(inst, perms, "ucddcp", d=d)), (n, extra)


@pytest.mark.parametrize("n", [17, 33, 64, 65, 100, 128, 129, 200, 256, 257, 300, 512, 513, 777,
                               999, 1000, 1023, 1024])
@pytest.mark.parametrize("pad", [0, 5, 8])
def test_ucddcp_batched_layouts(lib, n, pad):
    # ucddcp_eval_batch's several-sequences-per-warp kernel (8-byte table entries): every lane
    # layout, ragged tails (n % 8 != 0: the straddling chunk is patched in place) and garbage past
    # n; ld % 8 != 0 takes the warp-per-sequence kernel
    inst = gen.ucddcp_instance(n, 3 + n % 4)
    ld = gen.pad_ld(n) + pad
    perms = gen.random_perms(257, n, 500 + n + pad, ld=ld)
    perms[:, n:] = 4321
    for extra in (0, 1000):
        d = inst.sum_p + extra
        assert np.array_equal(_gpu_eval(lib, inst, perms, "ucddcp", d=d),
                              _oracle(inst, perms, "ucddcp", d=d)), (n, ld, extra)


@pytest.mark.parametrize("n", [20, 40, 300, 1000])
def test_ucddcp_wide_values(lib, n):
    # zero penalties, gamma = 0 and gamma up to the packed-record limit (127 with alpha, beta <= 7,
    # p <= 30): compression decisions on both sides of min(w, gamma)
    import dataclasses

    inst = gen.ranged_instance(n, 17, (1, 30), (0, 7), (0, 7), 1.0, problem="ucddcp")
    gamma = gen._uniform_int(gen._words(5, n, 26, n), 0, 127).astype(np.int32)
    inst = dataclasses.replace(inst, gamma=gamma)
    perms = gen.random_perms(300, n, n)
    assert np.array_equal(_gpu_eval(lib, inst, perms, "ucddcp"), _oracle(inst, perms, "ucddcp"))


def test_small_value_instances_and_zero_weights(lib):
    # tiny values, zero penalties, restrictive and unrestricted due dates
    for c in range(300):
        n = 1 + c % 40
        inst = gen.random_small(n, 9000 + c, pmax=7, wmax=4, zero_weights=(c % 3 == 0))
        perms = gen.random_perms(64, n, c)
        assert np.array_equal(_gpu_eval(lib, inst, perms), _oracle(inst, perms)), c
        if c % 2 == 0:
            d = inst.sum_p + c % 5
            assert np.array_equal(_gpu_eval(lib, inst, perms, "ucddcp", d=d),
                                  _oracle(inst, perms, "ucddcp", d=d)), c


def test_config2_shape_n100_all_h(lib):
    # BASELINE config 2 shape: n=100, h in {0.2,...,0.8}, 10 instances each (20k sequences each)
    perms = gen.random_perms(20000, 100, 2024)
    for k in range(1, 11):
        for h in gen.H_VALUES:
            inst = gen.cdd_instance(100, k, h)
            assert np.array_equal(_gpu_eval(lib, inst, perms), _oracle(inst, perms)), (k, h)


def test_unaligned_and_odd_stride(lib):
    import torch

    inst = gen.cdd_instance(100, 3, 0.4)
    perms = gen.random_perms(999, 100, 5, ld=103)  # ld % 8 != 0 -> scalar loads
    ref = _oracle(inst, perms)
    ins = lib.Instance.from_gen(inst)
    assert np.array_equal(lib.cdd_eval_batch(ins, _dev(perms)).cpu().numpy(), ref)
    big = torch.zeros((1000, 104), dtype=torch.int16, device="cuda")
    p8 = gen.random_perms(999, 100, 6, ld=104)
    big[1:, :] = _dev(p8)
    view = big[1:]  # 16-B aligned rows; also an unaligned base via a column offset
    assert np.array_equal(lib.cdd_eval_batch(ins, view).cpu().numpy(), _oracle(inst, p8))
    flat = torch.zeros(999 * 104 + 1, dtype=torch.int16, device="cuda")
    un = flat[1:].view(999, 104)
    un.copy_(_dev(p8))
    assert np.array_equal(lib.cdd_eval_batch(ins, un).cpu().numpy(), _oracle(inst, p8))


@pytest.mark.parametrize("n", [513, 600, 777, 1000, 1001, 1016, 1023, 1024])
@pytest.mark.parametrize("pad", [0, 3, 8, 16])
def test_large_n_row_strides(lib, n, pad):
    # 512 < n <= 1024 uses the 64-unit kernel: 256-bit loads when ld % 16 == 0, 128-bit when
    # ld % 8 == 0, scalar otherwise; straddling vectors when n % 8 != 0
    ld = n + pad
    if ld % 8 == 0 or pad == 3:
        inst = gen.cdd_instance(n, 2, 0.4)
        perms = gen.random_perms(333, n, n + pad, ld=ld)
        perms[:, n:] = 12345  # garbage past n must be ignored
        for h in (0.2, 0.8):
            d = int(h * inst.sum_p)
            assert np.array_equal(_gpu_eval(lib, inst, perms, d=d), _oracle(inst, perms, d=d)), (n, ld, h)


@pytest.mark.parametrize("n", [10, 50, 201, 500, 1000, 1023])
@pytest.mark.parametrize("problem", ["cdd", "ucddcp"])
def test_invalid_ids_flagged(lib, n, problem):
    inst = gen.ucddcp_instance(n, 1) if problem == "ucddcp" else gen.cdd_instance(n, 1, 0.4)
    ins = lib.Instance.from_gen(inst)
    fn = lib.ucddcp_eval_batch if problem == "ucddcp" else lib.cdd_eval_batch
    perms = gen.random_perms(70, n, 1)
    fn(ins, _dev(perms))
    lib.cdd_check(ins)  # valid rows: no flag
    npow2 = 1 << n.bit_length()
    for bad, pos in [(n, 7 % n), (npow2 - 1, n - 1), (32767, n // 2), (-1, 0)]:
        q = perms.copy()
        q[69 if bad == n else 3, pos] = bad
        fn(ins, _dev(q))
        with pytest.raises(lib.CddError) as e:
            lib.cdd_check(ins)
        assert e.value.code == lib.CDD_EDATA
        lib.cdd_check(ins)  # flag cleared


def test_host_e2e_path(lib):
    inst = gen.cdd_instance(1000, 1, 0.6)
    perms = gen.random_perms(3000, 1000, 8)
    ins = lib.Instance.from_gen(inst)
    out = lib.cdd_eval_batch_host(ins, perms)
    assert np.array_equal(out, _oracle(inst, perms))


def test_full_size_n1000_bench_launch(lib):
    # BASELINE metric configuration: n=1000, device-generated sequences (bench launch), sampled
    import torch

    inst = gen.cdd_instance(1000, 1, 0.4)
    ins = lib.Instance.from_gen(inst)
    perms = gen.random_perms_device(1 << 20, 1000, 99)
    out = lib.cdd_eval_batch(ins, perms)
    torch.cuda.synchronize()
    idx = np.random.default_rng(0).choice(perms.shape[0], 4000, replace=False)
    idx = np.concatenate([idx, [0, perms.shape[0] - 1]])
    sample = perms[torch.from_numpy(idx).cuda()].cpu().numpy()
    assert np.array_equal(out.cpu().numpy()[idx], _oracle(inst, sample))
    # property at full size: every penalty is within [min over sample-free bounds]: Z >= 0 and
    # Z <= (sum alpha + sum beta) * sum p
    o = out.cpu().numpy()
    assert (o >= 0).all() and (o <= (int(inst.alpha.sum()) + int(inst.beta.sum())) * inst.sum_p).all()


def test_instance_argument_errors(lib):
    with pytest.raises(lib.CddError):
        lib.Instance([0, 1], [1, 1], [1, 1], 3)          # p_i >= 1
    with pytest.raises(lib.CddError):
        lib.Instance([1] * 32768, [1] * 32768, [1] * 32768, 3)  # n <= 32767 (int16 job ids)
    with pytest.raises(lib.CddError) as e:  # a penalty could reach 2^62 (R20)
        lib.Instance([2**31 - 1] * 10, [2**31 - 1] * 10, [1] * 10, 3)
    assert e.value.code == lib.CDD_ERANGE
    # outside the packed records, inside int64: the generic path (round 1 refused these)
    assert lib.Instance([1000] * 10, [1000] * 10, [1] * 10, 3).query()["generic"]
    assert lib.Instance([1] * 1025, [1] * 1025, [1] * 1025, 3).query()["generic"]
    inst = gen.cdd_instance(20, 1, 0.4)
    ins = lib.Instance(inst.P, inst.alpha, inst.beta, inst.d)
    with pytest.raises(lib.CddError):
        lib.ucddcp_eval_batch(ins, _dev(gen.random_perms(4, 20, 1)))  # no UCDDCP data


@pytest.mark.parametrize("n", [40, 300, 313])
def test_cdd_weights_above_85(lib, n):
    # alpha, beta in (85, 100]: the batched evaluator takes the 16-bit pair pass (the byte-quad pass
    # needs max(alpha, beta) <= 85); one instance per side of the threshold (both on the fast path)
    for lo, hi in ((86, 100), (0, 85)):
        inst = gen.ranged_instance(n, 23 + lo, (1, 3), (lo, hi), (lo, hi), 0.4)
        ins = lib.Instance.from_gen(inst)
        assert not ins.wide
        perms = gen.random_perms(500, n, n + lo)
        assert np.array_equal(_gpu_eval(lib, inst, perms), _oracle(inst, perms)), (n, lo)
