"""CPU checks of the attention's KV-split planner (host logic behind tsv_attention_split_plan, used by
every attention launch of the step): the plan partitions the key tiles, fits the workspace it is
given, never loses to the unsplit launch in its own cost model, and attains the best modeled
makespan of its candidate family -- recomputed here by an independent list-scheduling simulation
(CTAs dispatched in block order to the first free SM; a CTA costs its key tiles + 2, a split range
+ 6; whole items first, then the tail's ranges, range-major)."""
import heapq

import pytest

SMS = 148
SLAB = lambda D: 128 * (D + 2) * 4   # noqa: E731  bytes of one query tile's (O, m, l) partial


@pytest.fixture(scope="module")
def tsv():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_asplos_luhtlwm0c26_b200 as m
    return m


def makespan(n_plain, plain_cost, n_tail, sizes, fixed=6, sms=SMS):
    free = [0.0] * sms
    for _ in range(n_plain):
        heapq.heapreplace(free, free[0] + plain_cost)
    for sz in sizes:                 # range-major: every tail item's range z before range z + 1
        for _ in range(n_tail):
            heapq.heapreplace(free, free[0] + sz + fixed)
    return max(free)


def best_in_family(L, H, D, ws_bytes, cnt_ints, sms=SMS, min_tiles=4, gain=0.97):
    n_all = -(-L // 128)
    C = -(-L // 256) * H
    base = makespan(C, n_all + 2, 0, [], sms=sms)
    best = base
    for S in range(2, 9):
        eq = -(-n_all // S)
        if eq < min_tiles:
            break
        sizes, left = [], n_all
        for _ in range(S):
            sizes.append(min(eq, left))
            left -= sizes[-1]
        if sizes[-1] < 1:
            continue
        for T in set(range(1, min(C, 3 * sms) + 1)) | {C}:
            if T * 2 * S * SLAB(D) > ws_bytes or T * 8 > cnt_ints:
                continue
            c = makespan(C - T, n_all + 2, T, sizes, sms=sms)
            if c < base * gain:
                best = min(best, c)
    return base, best


@pytest.mark.parametrize("L,H,D", [(16896, 3, 128), (16717, 3, 64), (4608, 12, 128), (4429, 6, 64), (1536, 12, 128),
                                   (600, 1, 64)])
def test_plan_is_the_best_of_its_family(tsv, L, H, D):
    ws, cnt = 128 << 20, 4096
    p = tsv.attention_split_plan(L, H, D, ws, cnt)
    n_all = -(-L // 128)
    C = -(-L // 256) * H
    assert p["n_plain"] + p["n_tail"] == C
    base, best = best_in_family(L, H, D, ws, cnt)
    if p["nsplit"] == 1:
        assert p["n_tail"] == 0 and best == base
        return
    b = p["bounds"]
    assert b[0] == 0 and b[-1] == n_all and all(y > x for x, y in zip(b, b[1:]))
    assert min(y - x for x, y in zip(b, b[1:])) >= 4
    assert p["n_tail"] * 2 * p["nsplit"] * SLAB(D) <= ws and p["n_tail"] * 8 <= cnt
    sizes = [y - x for x, y in zip(b, b[1:])]
    chosen = makespan(p["n_plain"], n_all + 2, p["n_tail"], sizes)
    assert chosen == best < 0.97 * base


def test_known_plans(tsv):
    # FLUX 2048^2 at SP = 1 (1584 items on 148 SMs): whole items only; at SP = 8 (198 items of 132
    # key tiles): a tail split whose modeled makespan beats both the unsplit launch (268) and the
    # uniform halves of round 2 (216 tile-times)
    assert tsv.attention_split_plan(16896, 24, 128, 128 << 20, 4096)["nsplit"] == 1
    p = tsv.attention_split_plan(16896, 3, 128, 128 << 20, 4096)
    sizes = [y - x for x, y in zip(p["bounds"], p["bounds"][1:])]
    assert 0 < p["n_plain"] < 198
    assert makespan(p["n_plain"], 134, p["n_tail"], sizes) < makespan(0, 0, 198, [66, 66]) == 216


def test_workspace_bounds_the_tail(tsv):
    # a workspace for 7 split blocks x 2 ranges: whatever the plan, its partials fit
    D = 128
    ws = 7 * 2 * 2 * SLAB(D)
    for L, H in ((4608, 12), (16896, 3), (16896, 6)):
        p = tsv.attention_split_plan(L, H, D, ws, 56)
        assert p["n_tail"] * 2 * p["nsplit"] * SLAB(D) <= ws or p["nsplit"] == 1
        assert p["n_tail"] * 8 <= 56 or p["nsplit"] == 1
    # no workspace at all: no split
    assert tsv.attention_split_plan(16896, 3, 128, 0, 0)["nsplit"] == 1


@pytest.mark.parametrize("nsplit", [2, 3, 8])
def test_forced_uniform_split(tsv, nsplit):
    L, H, D = 1000, 3, 128
    p = tsv.attention_split_plan(L, H, D, 64 << 20, 4096, nsplit=nsplit)
    n_all = -(-L // 128)
    assert p["n_plain"] == 0 and p["n_tail"] == -(-L // 256) * H
    tps = -(-n_all // nsplit)
    assert p["bounds"] == list(range(0, n_all, tps)) + [n_all]


def test_arguments(tsv):
    with pytest.raises(tsv.TsvError):
        tsv.attention_split_plan(0, 3, 128, 1 << 20, 64)
    with pytest.raises(tsv.TsvError):
        tsv.attention_split_plan(1000, 3, 96, 1 << 20, 64)
