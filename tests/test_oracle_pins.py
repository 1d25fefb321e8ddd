"""Pins of the CPU oracle against things other than itself.

Every function of oracle/ is checked here against what PAPER.md and the
MPI matching rules fix, never against a retyped copy of its own loop:

* brute-force enumeration of ALL partial injective receive->message maps on
  tiny queues, filtered by the four matching rules (admissibility, the two
  MPI non-overtaking rules with the arrival order of PAPER.md §II.B l.65, and
  progress) -- exactly one survivor, equal to the oracle's answer;
* the paper's own Algorithms 1 (multi-warp ballot scan) and 2 (column
  reduce) (§V.A l.151-173), a different algorithm from the two-list
  traversal, executed literally;
* the theorem of DESIGN.md §2.2: any interleaving of posts and arrivals
  gives the same matching, so the batch equals the event-driven engine;
* hand-worked golden cases (tests/golden/*.json);
* closed forms for the relaxations (n-th receive of a key <-> n-th message of
  that key; per-key match count = min(#recv_k, #msg_k)).
"""
import itertools
import json
import os

import numpy as np
import pytest

import oracle
import synth

ANY_S, ANY_T = synth.ANY_SOURCE, synth.ANY_TAG
GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def fields(h):
    h = int(h)
    return h & 0xFFFFFFFF, (h >> 32) & 0xFFFF, (h >> 48) & 0xFFFF


def admits(r, m):
    """PAPER.md §II.B l.65: (src, tag, comm), ANY_SOURCE / ANY_TAG on receives."""
    rs, rt, rc = fields(r)
    ms, mt, mc = fields(m)
    return rc == mc and (rs == ANY_S or rs == ms) and (rt == ANY_T or rt == mt)


def mpi_rules_hold(R, M, pi):
    """The matching rules, stated declaratively (pi: dict recv -> msg).

    (A) admissible pairs (l.65);
    (B) receive-side non-overtaking (MPI-3.1 §3.5): if R_i < R_i' both admit
        M_j and M_j went to R_i', then R_i was satisfied before it, i.e. by an
        earlier-arrived message;
    (C) message-side order, strengthened to the single arrival order of one
        queue (north_star: "the earliest-arrived unmatched message it
        admits"): if M_j < M_j' both are admitted by R_i and M_j' went to R_i,
        then M_j went to an earlier receive;
    (D) progress: no unmatched receive admits an unmatched message."""
    inv = {j: i for i, j in pi.items()}
    for i, j in pi.items():
        if not admits(R[i], M[j]):
            return False
    for i2, j in pi.items():
        for i in range(i2):
            if admits(R[i], M[j]) and not (i in pi and pi[i] < j):
                return False
    for i, j2 in pi.items():
        for j in range(j2):
            if admits(R[i], M[j]) and not (j in inv and inv[j] < i):
                return False
    for i in range(len(R)):
        if i in pi:
            continue
        for j in range(len(M)):
            if j not in inv and admits(R[i], M[j]):
                return False
    return True


def all_partial_injections(nr, nm):
    for k in range(min(nr, nm) + 1):
        for rs in itertools.combinations(range(nr), k):
            for ms in itertools.permutations(range(nm), k):
                yield dict(zip(rs, ms))


def tiny_case(rng, nr, nm, p_wild=0.35):
    src = rng.integers(0, 2, nr + nm)
    tag = rng.integers(0, 2, nr + nm)
    comm = rng.integers(0, 2, nr + nm) * (rng.random() < 0.3)
    R = synth.pack(np.where(rng.random(nr) < p_wild, ANY_S, src[:nr]),
                   np.where(rng.random(nr) < p_wild, ANY_T, tag[:nr]), comm[:nr])
    M = synth.pack(src[nr:], tag[nr:], comm[nr:])
    return R, M


@pytest.mark.parametrize("seed", range(60))
def test_mpi_bruteforce_unique_and_equal(seed):
    rng = np.random.default_rng(seed)
    nr, nm = int(rng.integers(0, 5)), int(rng.integers(0, 5))
    R, M = tiny_case(rng, nr, nm)
    sols = [pi for pi in all_partial_injections(nr, nm) if mpi_rules_hold(R, M, pi)]
    assert len(sols) == 1, "the matching rules must define a unique assignment"
    mr, mm = oracle.mpi_two_list(R, M)
    got = {i: int(j) for i, j in enumerate(mr) if j >= 0}
    assert got == sols[0]
    for i, j in got.items():
        assert mm[j] == i
    assert (mm >= 0).sum() == len(got)


@pytest.mark.parametrize("seed", range(40))
def test_mpi_bruteforce_wide_fields_and_literal_any(seed):
    """As above with full-width field values (src near 2^32, tag near 2^16,
    16-bit communicators) and messages that carry the reserved wildcard
    values themselves (reading R2: matched literally -- only a receive whose
    field is the wildcard admits them)."""
    rng = np.random.default_rng(7000 + seed)
    nr, nm = int(rng.integers(0, 5)), int(rng.integers(0, 5))
    sv = np.array([ANY_S, 0xFFFFFFFE, 0x80000000], dtype=np.uint64)
    tv = np.array([ANY_T, 0xFFFE, 0x8000], dtype=np.uint64)
    cv = np.array([0xFFFF, 0x8001], dtype=np.uint64)
    R = synth.pack(sv[rng.integers(0, 3, nr)], tv[rng.integers(0, 3, nr)], cv[rng.integers(0, 2, nr)])
    M = synth.pack(sv[rng.integers(0, 3, nm)], tv[rng.integers(0, 3, nm)], cv[rng.integers(0, 2, nm)])
    sols = [pi for pi in all_partial_injections(nr, nm) if mpi_rules_hold(R, M, pi)]
    assert len(sols) == 1
    mr, _ = oracle.mpi_two_list(R, M)
    assert {i: int(j) for i, j in enumerate(mr) if j >= 0} == sols[0]


def paper_algorithms_1_2(R, M, warp=4):
    """PAPER.md §V.A, executed literally.  Algorithm 1 (l.151-158): thread t
    holds message t, for every receive i a warp ballots SendObj == RecvObj and
    writes the vote to voteMatrix[warp_id * window + i].  Algorithm 2
    (l.160-173): one warp, thread t < warps reads the votes of row t, bidders =
    ballot(vote & mask), the lowest bidder thread takes ffs(vote & mask) - 1,
    clears it from its mask, and result[i] = thread_id * warp_size + match.
    The object comparison is the MPI admission of l.65."""
    n_warps = max(1, -(-len(M) // warp))
    assert n_warps <= warp, "Algorithm 2 reduces with a single warp"
    window = len(R)
    vote = np.zeros(n_warps * max(window, 1), dtype=np.int64)
    for w in range(n_warps):                       # Algorithm 1
        for i in range(window):
            v = 0
            for lane in range(warp):
                t = w * warp + lane
                if t < len(M) and admits(R[i], M[t]):
                    v |= 1 << lane
            vote[w * window + i] = v
    result = [-1] * window
    mask = [(1 << warp) - 1] * warp                # Algorithm 2, per thread
    for i in range(window):
        votes = [int(vote[t * window + i]) if t < n_warps else 0 for t in range(warp)]
        bidders = [t for t in range(warp) if votes[t] & mask[t]]
        if not bidders:
            continue
        t = bidders[0]                             # ffs(bidders) - 1
        x = votes[t] & mask[t]
        match = (x & -x).bit_length() - 1          # ffs(vote & mask) - 1
        mask[t] &= ~(1 << match)
        result[i] = t * warp + match
    return result


@pytest.mark.parametrize("seed", range(25))
@pytest.mark.parametrize("warp", [4, 8])
def test_mpi_equals_paper_algorithms_1_2(seed, warp):
    rng = np.random.default_rng(1000 + seed)
    cap = warp * warp
    nr, nm = int(rng.integers(0, cap + 1)), int(rng.integers(0, cap + 1))
    src = rng.integers(0, 3, nr + nm)
    tag = rng.integers(0, 3, nr + nm)
    R = synth.pack(np.where(rng.random(nr) < 0.25, ANY_S, src[:nr]),
                   np.where(rng.random(nr) < 0.25, ANY_T, tag[:nr]))
    M = synth.pack(src[nr:], tag[nr:])
    mr, _ = oracle.mpi_two_list(R, M)
    assert list(mr) == paper_algorithms_1_2(R, M, warp)


def test_mpi_config0_equals_paper_algorithms_1_2():
    q = synth.mpi_small(0)
    mr, _ = oracle.mpi_two_list(q.recv_hdr, q.msg_hdr)
    assert list(mr) == paper_algorithms_1_2(q.recv_hdr, q.msg_hdr, warp=8)


@pytest.mark.parametrize("seed", range(20))
def test_mpi_interleaving_invariance(seed):
    """DESIGN.md §2.2 theorem: with per-side orders fixed, every interleaving
    of receive posts and message arrivals yields the same matching."""
    rng = np.random.default_rng(2000 + seed)
    R, M = tiny_case(rng, int(rng.integers(0, 30)), int(rng.integers(0, 30)))
    base = oracle.mpi_two_list(R, M)
    for _ in range(6):
        kinds = rng.permutation(np.r_[np.zeros(len(R), int), np.ones(len(M), int)])
        ev, i, j = [], 0, 0
        for k in kinds:
            if k == 0:
                ev.append(i); i += 1
            else:
                ev.append(-j - 1); j += 1
        got = oracle.mpi_two_list(R, M, events=ev)
        assert np.array_equal(got[0], base[0]) and np.array_equal(got[1], base[1])


def check_invariants(R, M, mr, mm):
    """Rules (A)-(D) of mpi_rules_hold, vectorised for medium sizes."""
    nr, nm = len(R), len(M)
    A = np.array([[admits(r, m) for m in M] for r in R], dtype=bool).reshape(nr, nm)
    got = {i: int(j) for i, j in enumerate(mr) if j >= 0}
    inv = {j: i for i, j in got.items()}
    assert len(inv) == len(got), "a message matched twice"
    for j, i in enumerate(mm):
        assert (i < 0 and j not in inv) or inv.get(j) == i
    for i, j in got.items():
        assert A[i, j]
        earlier = np.nonzero(A[i, :j])[0]
        assert all(k in inv and inv[k] < i for k in earlier), "non-overtaking (msg)"
        ri = np.nonzero(A[:i, j])[0]
        assert all(k in got and got[k] < j for k in ri), "non-overtaking (recv)"
    free_m = np.array([j not in inv for j in range(nm)], dtype=bool)
    for i in range(nr):
        if i not in got and nm:
            assert not (A[i] & free_m).any(), "progress"


@pytest.mark.parametrize("seed", range(8))
def test_mpi_invariants_medium(seed):
    q = synth.random_case(seed, n_ep=4, max_depth=120)
    for e in range(q.n_endpoints):
        R, M = q.endpoint(e)
        mr, mm = oracle.mpi_two_list(R, M)
        check_invariants(R, M, mr, mm)


def test_mpi_golden_cases():
    with open(os.path.join(GOLDEN, "mpi_cases.json")) as f:
        cases = json.load(f)["cases"]
    assert len(cases) >= 4
    for c in cases:
        R = synth.pack([ANY_S if s == "ANY" else s for s, t, k in c["recv"]],
                       [ANY_T if t == "ANY" else t for s, t, k in c["recv"]],
                       [k for s, t, k in c["recv"]])
        M = synth.pack([s for s, t, k in c["msg"]], [t for s, t, k in c["msg"]],
                       [k for s, t, k in c["msg"]])
        mr, _ = oracle.mpi_two_list(R, M)
        assert list(mr) == c["expect_recv_to_msg"], c["name"]


def test_mpi_endpoints_equal_per_endpoint():
    q = synth.random_case(7, n_ep=6, max_depth=50)
    mr, mm = oracle.mpi_endpoints(q)
    for e in range(q.n_endpoints):
        R, M = q.endpoint(e)
        a, b = oracle.mpi_two_list(R, M)
        r0, m0 = q.recv_off[e], q.msg_off[e]
        assert np.array_equal(np.where(a >= 0, a + m0, -1), mr[r0:r0 + len(R)])
        assert np.array_equal(np.where(b >= 0, b + r0, -1), mm[m0:m0 + len(M)])


@pytest.mark.parametrize("sem", [oracle.SEM_MPI, oracle.SEM_NOWILD_ORDERED])
@pytest.mark.parametrize("seed", range(6))
def test_batches_compose(sem, seed):
    """Matching split into batches (residual queues carried over) yields the
    same pairs as one batch over everything (the final
    matching is interleaving-invariant, batches are one interleaving)."""
    rng = np.random.default_rng(3000 + seed)
    wild = sem == oracle.SEM_MPI
    q = synth.random_case(seed, n_ep=3, max_depth=60, wild=wild)
    one = oracle.OracleEngine(sem, q.n_endpoints)
    one.post_recvs(q.recv_hdr, None, q.recv_off)
    one.push_msgs(q.msg_hdr, None, q.msg_off)
    r_all, m_all = one.match_batch()
    ref = {int(r): int(m) for r, m in zip(r_all, m_all) if m >= 0}
    eng = oracle.OracleEngine(sem, q.n_endpoints)
    # split every endpoint's queues at random points into three batches
    cuts_r = [np.sort(rng.integers(q.recv_off[e], q.recv_off[e + 1] + 1, 2)) for e in range(q.n_endpoints)]
    cuts_m = [np.sort(rng.integers(q.msg_off[e], q.msg_off[e + 1] + 1, 2)) for e in range(q.n_endpoints)]
    got = {}
    for b in range(3):
        def piece(off, cuts, hdr):
            hs, cs, o = [], [], [0]
            for e in range(q.n_endpoints):
                bounds = [off[e], *cuts[e], off[e + 1]]
                lo, hi = int(bounds[b]), int(bounds[b + 1])
                hs.append(hdr[lo:hi]); cs.append(np.arange(lo, hi)); o.append(o[-1] + hi - lo)
            return np.concatenate(hs), np.concatenate(cs), o
        h, c, o = piece(q.recv_off, cuts_r, q.recv_hdr)
        eng.post_recvs(h, c, o)
        h, c, o = piece(q.msg_off, cuts_m, q.msg_hdr)
        eng.push_msgs(h, c, o)
        r, m = eng.match_batch()
        for rc, mc in zip(r, m):
            if mc >= 0:
                assert int(rc) not in got
                got[int(rc)] = int(mc)
    assert got == ref


# --------------------------------------------------------------- relaxations


def rank_pairing(R, M):
    """Closed form of the ordered no-wildcard mode: per identical tuple, the
    n-th posted receive takes the n-th arrived message."""
    by_key = {}
    for j, m in enumerate(M):
        by_key.setdefault(int(m), []).append(j)
    seen = {}
    out = []
    for r in R:
        k = int(r)
        n = seen.get(k, 0)
        seen[k] = n + 1
        lst = by_key.get(k, [])
        out.append(lst[n] if n < len(lst) else -1)
    return out


@pytest.mark.parametrize("seed", range(12))
def test_nowild_ordered_closed_form(seed):
    q = synth.random_case(100 + seed, n_ep=1, max_depth=300, wild=False, n_src=5, n_tag=3)
    R, M = q.endpoint(0)
    mr, mm = oracle.nowild_ordered(R, M)
    assert list(mr) == rank_pairing(R, M)
    assert sorted(j for j in mm if j >= 0) == sorted(i for i, j in enumerate(mr) if j >= 0)


@pytest.mark.parametrize("seed", range(6))
def test_nowild_ordered_equals_mpi_without_wildcards(seed):
    q = synth.nowild_pairs(seed, n=3000, n_src=20, n_tag=8, p_unmatched=0.1)
    a = oracle.nowild_ordered(q.recv_hdr, q.msg_hdr)
    b = oracle.mpi_two_list(q.recv_hdr, q.msg_hdr)
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])


def test_nowild_wildcard_values_are_literal():
    R = synth.pack([ANY_S, 3, 3], [5, ANY_T, 5])
    M = synth.pack([3, ANY_S, 3], [5, 5, ANY_T])
    mr, _ = oracle.nowild_ordered(R, M)
    assert list(mr) == [1, 2, 0]
    mr, _ = oracle.nowild_unordered(R, M)
    assert list(mr) == [1, 2, 0]


def key_counts(R, M, mr):
    from collections import Counter
    cr, cm = Counter(map(int, R)), Counter(map(int, M))
    got = Counter(int(R[i]) for i, j in enumerate(mr) if j >= 0)
    return cr, cm, got


def check_unordered_valid(R, M, mr, mm):
    got = {i: int(j) for i, j in enumerate(mr) if j >= 0}
    assert len(set(got.values())) == len(got)
    for i, j in got.items():
        assert int(R[i]) == int(M[j]) and mm[j] == i
    assert (mm >= 0).sum() == len(got)
    cr, cm, per = key_counts(R, M, mr)
    for k in set(cr) | set(cm):
        assert per.get(k, 0) == min(cr.get(k, 0), cm.get(k, 0)), "maximal per key"


@pytest.mark.parametrize("seed", range(12))
def test_nowild_unordered_valid_and_maximal(seed):
    q = synth.random_case(200 + seed, n_ep=1, max_depth=400, wild=False, n_src=6, n_tag=4)
    R, M = q.endpoint(0)
    mr, mm = oracle.nowild_unordered(R, M)
    check_unordered_valid(R, M, mr, mm)


def test_nowild_unordered_perfect_match_all_matched():
    q = synth.nowild_pairs(5, n=20000, n_src=300, n_tag=40)
    mr, mm, it = oracle.nowild_unordered(q.recv_hdr, q.msg_hdr, return_iterations=True)
    assert (mr >= 0).all() and (mm >= 0).all()
    check_unordered_valid(q.recv_hdr, q.msg_hdr, mr, mm)
    assert it >= 1


def _fold(h):
    """The 64-bit header folded to the paper's 32-bit key (reading R7)."""
    hv = int(h)
    return oracle.jenkins32((hv & 0xFFFFFFFF) ^ oracle.jenkins32(hv >> 32))


def _same_primary_keys(n, P, want_sec=None, S=1):
    """n distinct tuples whose primary slots (fold % P) coincide; with
    want_sec, the i-th key's secondary slot (J(fold) % S) is want_sec[i]."""
    keys, target, k = [], None, 0
    while len(keys) < n:
        h = synth.pack(k, 1)
        f = _fold(h)
        if target is None:
            target = f % P
        if f % P == target and (want_sec is None or oracle.jenkins32(f) % S == want_sec[len(keys)]):
            keys.append(h)
        k += 1
    return np.array(keys, dtype=np.uint64)


def test_nowild_unordered_collisions_are_held():
    """PAPER.md §VI.C l.219, worked by hand.  Three receives (S = 1, P = 5,
    reading R8) whose primary slots collide, messages in reverse order.
    Iteration 1: R0 -> primary, R1 -> secondary (first collision), R2 held
    (second collision); M(R2) finds neither and is deferred, M(R1) hits the
    secondary, M(R0) the primary.  Iteration 2: R2 -> primary, M(R2) hits.
    Exactly 2 iterations -- without the secondary table it would take 3
    (one receive tabled per iteration)."""
    R = _same_primary_keys(3, 5)
    M = R[::-1].copy()
    mr, mm, it = oracle.nowild_unordered(R, M, return_iterations=True)
    assert it == 2
    assert (mr >= 0).all()
    check_unordered_valid(R, M, mr, mm)


def test_nowild_unordered_secondary_slot_is_second_hash():
    """Five receives (S = 2, P = 10) on one primary slot; R1 and R2 have
    different secondary slots J(key) % 2 (reading R7), R3 and R4 then collide
    twice.  Iteration 1 tables R0 (primary), R1 and R2 (both secondary
    slots); messages in reverse order match R2, R1, R0 and defer M(R4),
    M(R3).  Iteration 2 tables R3 (primary) and R4 (the freed secondary
    slot) and both match: exactly 2 iterations.  A secondary slot taken from
    the primary hash (key % 2, equal for all five since key % 10 is) would
    hold R2 and need 3; no secondary table, 5."""
    R = _same_primary_keys(5, 10, want_sec=[0, 0, 1, 0, 1], S=2)
    M = R[::-1].copy()
    mr, mm, it = oracle.nowild_unordered(R, M, return_iterations=True)
    assert it == 2
    assert (mr >= 0).all()
    check_unordered_valid(R, M, mr, mm)


@pytest.mark.parametrize("seed", range(25))
def test_nowild_unordered_bruteforce(seed):
    """On tiny queues the oracle's answer is one of the maximum matchings of
    equal tuples found by exhaustive enumeration."""
    rng = np.random.default_rng(4000 + seed)
    nr, nm = int(rng.integers(0, 5)), int(rng.integers(0, 5))
    R = synth.pack(rng.integers(0, 2, nr), rng.integers(0, 2, nr))
    M = synth.pack(rng.integers(0, 2, nm), rng.integers(0, 2, nm))
    valid = [pi for pi in all_partial_injections(nr, nm)
             if all(int(R[i]) == int(M[j]) for i, j in pi.items())]
    best = max(len(pi) for pi in valid)
    mr, _ = oracle.nowild_unordered(R, M)
    got = {i: int(j) for i, j in enumerate(mr) if j >= 0}
    assert got in valid and len(got) == best


def test_jenkins32_known_answers():
    """Known-answer vectors for the paper's hash (§VI.C l.219, ref.
    [17]: Jenkins' 32-bit 6-shift integer hash), worked line by line from the
    published listing outside oracle/ (tests/golden/jenkins32.json, with its
    worksheet).  A wrong constant or shift in any of the six lines changes
    these outputs."""
    doc = json.load(open(os.path.join(GOLDEN, "jenkins32.json")))
    assert len(doc["vectors"]) >= 4
    for v in doc["vectors"]:
        assert oracle.jenkins32(int(v["in"], 16)) == int(v["steps"][-1], 16), v["in"]


def test_jenkins_is_a_bijection_sample():
    """Each of the six steps is invertible, so the hash permutes 2^32; a
    collision on a sample would reveal a typo in a constant or shift."""
    xs = np.random.default_rng(9).choice(1 << 32, 20000, replace=False)
    hs = {oracle.jenkins32(int(x)) for x in xs}
    assert len(hs) == len(xs)


@pytest.mark.parametrize("seed,kind,msg_frac,p_after", [(1, "src", 1.0, 0.05), (2, "tag", 0.6, 0.2),
                                                         (3, "src", 0.4, 0.0), (4, "tag", 1.0, 0.3)])
def test_leading_wildcard_run_takes_group_messages_in_arrival_order(seed, kind, msg_frac, p_after):
    """The reading behind the kernel's leading-run merge,
    checked on the oracle: wildcards of one type posted before any exact
    receive their group admits see no competing claim, so the r-th of them
    takes the r-th admissible message in arrival order (§II.B
    l.65-67: earliest unmatched message, receives in posting order), or
    nothing once the group's messages are used up."""
    q = synth.lead_runs(seed, n_ep=3, depth=600, lead=200, kind=kind, msg_frac=msg_frac, p_wild_after=p_after,
                        n_src=6, n_tag=4, ragged=True)
    mr, _ = oracle.mpi_endpoints(q)
    src = (q.recv_hdr & 0xFFFFFFFF).astype(np.int64)
    tag = ((q.recv_hdr >> 32) & 0xFFFF).astype(np.int64)
    msrc = (q.msg_hdr & 0xFFFFFFFF).astype(np.int64)
    mtag = ((q.msg_hdr >> 32) & 0xFFFF).astype(np.int64)
    checked = 0
    for e in range(q.n_endpoints):
        r0, r1, m0, m1 = q.recv_off[e], q.recv_off[e + 1], q.msg_off[e], q.msg_off[e + 1]
        wild = (src[r0:r1] == synth.ANY_SOURCE) if kind == "src" else (tag[r0:r1] == synth.ANY_TAG)
        gkey_r = tag[r0:r1] if kind == "src" else src[r0:r1]
        gkey_m = mtag[m0:m1] if kind == "src" else msrc[m0:m1]
        mtuples = set(zip(msrc[m0:m1].tolist(), mtag[m0:m1].tolist()))
        for gval in np.unique(gkey_r[wild]):
            # first exact receive admitting one of the group's messages
            fe = r1 - r0
            for i in range(r1 - r0):
                if not wild[i] and gkey_r[i] == gval and (src[r0 + i], tag[r0 + i]) in mtuples:
                    fe = i
                    break
            run = [i for i in range(fe) if wild[i] and gkey_r[i] == gval]
            gmsgs = [m0 + j for j in range(m1 - m0) if gkey_m[j] == gval]
            for r, i in enumerate(run):
                want = gmsgs[r] if r < len(gmsgs) else -1
                assert mr[r0 + i] == want, (e, gval, r)
                checked += 1
    assert checked > 100
