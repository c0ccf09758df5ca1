"""Model check of the fused peer-memory exchange protocol (csrc/peer.cuh) on CPU.

Each rank runs, per tree and level, the stream-ordered steps of the peer path:
  find_split   writes keys[L] of its own window
  split_record publishes flag_keys = E, waits for every peer's flag_keys >= E, reads keys[L]
               of every window, writes records + bitmap into xchg[L] of its own window
  partition    publishes flag_rec = E, waits for every peer's flag_rec >= E, reads xchg[L] of
               every window; then the plan kernel advances the epoch (E = epoch + 1)
Ranks advance in random interleavings (a blocked wait yields).  Every read must see exactly the
version written for the same (tree, level): no rank may overwrite a buffer a peer has yet to read.
The two flags make even a single buffer per kind safe (a rank rewrites keys only after the peers
published flag_rec, i.e. finished reading them, and xchg only after they published the next
flag_keys); the library keeps one per level anyway.  The checker flags the race of a protocol
without the second flag, so it is able to see the failure it rules out."""
import random

import pytest


def _simulate(N, D, T, seed, buffer_of, second_flag=True):
    rng = random.Random(seed)
    win = [{"fk": 0, "fr": 0, "keys": {}, "xchg": {}} for _ in range(N)]
    epoch = [0] * N

    def program(r):
        for t in range(T):
            for L in range(D):
                yield ("write", "keys", buffer_of(t, L), (t, L))
                yield ("publish", "fk")
                yield ("wait", "fk")
                for p in range(N):
                    yield ("read", p, "keys", buffer_of(t, L), (t, L))
                yield ("write", "xchg", buffer_of(t, L), (t, L))
                if second_flag:
                    yield ("publish", "fr")
                    yield ("wait", "fr")
                for p in range(N):
                    yield ("read", p, "xchg", buffer_of(t, L), (t, L))
                yield ("epoch",)

    progs = [program(r) for r in range(N)]
    pending = [next(p) for p in progs]
    done = [False] * N
    bad = []
    while not all(done):
        r = rng.choice([i for i in range(N) if not done[i]])
        op = pending[r]
        E = epoch[r] + 1
        if op[0] == "wait":
            if any(win[p][op[1]] < E for p in range(N) if p != r):
                continue                         # blocked: another rank runs
        elif op[0] == "publish":
            win[r][op[1]] = E
        elif op[0] == "write":
            win[r][op[1]][op[2]] = op[3]
        elif op[0] == "read":
            _, p, kind, buf, want = op
            got = win[p][kind].get(buf)
            if got != want:
                bad.append((r, p, kind, want, got))
        elif op[0] == "epoch":
            epoch[r] += 1
        try:
            pending[r] = next(progs[r])
        except StopIteration:
            done[r] = True
    return bad, epoch


@pytest.mark.parametrize("N", [2, 3, 8])
@pytest.mark.parametrize("D", [1, 2, 3, 5, 8])
@pytest.mark.parametrize("layout", ["per_level", "single"])
def test_exchange_is_race_free(N, D, layout):
    buf = (lambda t, L: L) if layout == "per_level" else (lambda t, L: 0)
    for seed in range(40):
        bad, epoch = _simulate(N, D, T=3, seed=seed, buffer_of=buf)
        assert not bad, bad[:3]
        assert epoch == [3 * D] * N


def test_checker_sees_race_without_second_flag():
    """Without flag_rec a rank reads the peers' records while they may not be written yet (or
    already overwritten by the next level)."""
    hits = 0
    for seed in range(100):
        bad, _ = _simulate(2, 3, T=3, seed=seed, buffer_of=lambda t, L: L, second_flag=False)
        hits += bool(bad)
    assert hits > 0
