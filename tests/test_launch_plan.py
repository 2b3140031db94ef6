"""CPU tests of the launch-plan host logic (uc_jacobi_launch_plan): how uc_jacobi_run splits
`iters` iterations into kernel launches of 1..T iterations (variants 4 and 5).  The multi-
iteration kernels are only correct under these rules, so the plan is checked
against them for every starting iteration k, and against a direct Python restatement."""
import itertools

import pytest

U = pytest.importorskip("paper_conf_cluster_sagbilieinu25_b200")

DEV, HOST, PARTIAL = U.UC_MODE_DEVICE, U.UC_MODE_HOST, U.UC_MODE_PARTIAL


def restated(variant, levels, mode, n, iters, ne):
    """The rules, written out independently of the C++."""
    if variant == 5:
        plan, i = [], 0
        while i < iters:
            t = min(levels, iters - i)
            while t > 1 and not (mode == DEV and n >= 2 * t and (ne <= 0 or ne >= t)):
                t -= 1
            plan.append(t)
            i += t
        if len(plan) >= 2 and plan[-1] < plan[-2] - 1:  # even split of a short remainder
            tot = plan[-2] + plan[-1]
            plan[-2:] = [(tot + 1) // 2, tot // 2]
        return plan
    if variant == 4 and mode == DEV and n >= 2 and ne != 1:
        return [2] * (iters // 2) + [1] * (iters % 2)
    return [1] * iters


CASES = list(itertools.product([1, 4, 5], [1, 2, 3, 4, 6, 8], [DEV, HOST, PARTIAL], [1, 2, 3, 4, 7, 8, 15, 16, 16384]))


@pytest.mark.parametrize("variant,levels,mode,n", CASES)
def test_plan_rules(variant, levels, mode, n):
    for ne in (0, 1, 2, 3, 4, 5, 7, 100):
        for iters in (0, 1, 2, 3, 5, 8, 99, 100, 101):
            plan = U.launch_plan(variant, levels, mode, n, iters, ne)
            assert plan == restated(variant, levels, mode, n, iters, ne)
            assert sum(plan) == iters and all(t >= 1 for t in plan)
            cap = levels if variant == 5 else (2 if variant == 4 else 1)
            assert all(t <= cap for t in plan)
            for t in plan:
                if t > 1:
                    # multi-iteration launches: fused device mode only, every boundary round inside
                    # the slab, at most one norm round in the launch for ANY starting k
                    assert mode == DEV
                    assert n >= (2 * t if variant == 5 else 2)
                    for k0 in range(0, 2 * max(ne, 1) + 1):
                        norms = sum(1 for kk in range(k0, k0 + t) if ne > 0 and kk % ne == 0)
                        assert norms <= 1
            # greedy: only the last two launches of a run may be shorter than the deepest feasible
            # one, and they differ by at most 1 after the split of a short remainder
            if variant == 5 and plan:
                assert all(t == plan[0] for t in plan[:-2]) and all(t <= plan[0] for t in plan)
                if len(plan) >= 2:
                    assert plan[-1] >= plan[-2] - 1


def test_bench_configuration_plan():
    """The default bench step: 100 iterations, norm every 100, 16384 rows -> 25 launches of 4."""
    assert U.launch_plan(5, 4, DEV, 16384, 100, 100) == [4] * 25
    assert U.launch_plan(5, 4, DEV, 2048, 100, 100) == [4] * 25    # configs[2] slab at P = 8
    assert U.launch_plan(5, 4, DEV, 6, 10, 0) == [3, 3, 2, 2]       # n = 6: T' = 3 (3 + 1 split)
    assert U.launch_plan(5, 4, DEV, 16384, 10, 3) == [3, 3, 2, 2]   # norm every 3 < T
    assert U.launch_plan(5, 4, HOST, 16384, 3, 0) == [1, 1, 1]
    assert U.launch_plan(4, 0, DEV, 16384, 5, 0) == [2, 2, 1]      # variant 4: pairs + 1
    # two ghost lanes (T up to 8): 100 = 11 x 8 + 6 + 6 (the short remainder 4 is split evenly)
    assert U.launch_plan(5, 8, DEV, 16384, 100, 100) == [8] * 11 + [6, 6]
    assert U.launch_plan(5, 6, DEV, 16384, 100, 100) == [6] * 15 + [5, 5]
    assert U.launch_plan(5, 8, DEV, 16384, 9, 0) == [5, 4]
    # deep-halo host mode follows the device plan; the paper's host path is one per launch
    assert U.launch_plan(5, 6, HOST | U.UC_PLAN_DEEP_HALO, 16384, 13, 6) == [6, 4, 3]
    assert U.launch_plan(5, 6, DEV, 16384, 1000, 100) == [6] * 165 + [5, 5]  # configs[1]
    assert U.launch_plan(5, 6, HOST, 16384, 3, 0) == [1, 1, 1]
    assert U.launch_plan(5, 8, DEV, 10, 100, 0) == [5] * 20           # n = 10: T' = 5


def test_plan_argument_errors():
    with pytest.raises(U.UCError):
        U.launch_plan(5, 9, DEV, 100, 10, 0)
    with pytest.raises(U.UCError):
        U.launch_plan(5, 4, DEV, 0, 10, 0)
