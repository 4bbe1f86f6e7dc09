"""T3: the claim protocol of cycle_global.cu under random interleavings (tools/protocol_sim.py).
The kernel's protocol must never corrupt; the two known-wrong variants must be caught."""
import itertools

from tools.protocol_sim import simulate

SHAPES = [(2, 3), (3, 5), (5, 3), (4, 4), (6, 6), (3, 8), (7, 7), (8, 12)]


def test_p1_never_corrupts():
    for (A, B), workers, seed in itertools.product(SHAPES, [2, 3, 8, 64], range(30)):
        ok, _ = simulate(A, B, "P1", workers, seed)
        assert ok, (A, B, workers, seed)


def _fails_somewhere(protocol):
    for (A, B), workers, seed in itertools.product(SHAPES, [2, 3, 8, 64], range(30)):
        ok, _ = simulate(A, B, protocol, workers, seed)
        if not ok:
            return True
    return False


def test_p0_without_recheck_is_caught():
    assert _fails_somewhere("P0")


def test_unclaimed_cycle_close_is_caught():
    """The square-matrix bug: closing a cycle at the walker's own start without claiming."""
    assert _fails_somewhere("HOME_SKIP")


def test_single_walker_is_sequential_cycle_following():
    ok, st = simulate(5, 3, "P1", 1, 0)
    assert ok
    # 5x3: 15 elements, 3 fixed points -> 12 moved; each written exactly once
    assert st["writes"] == 12
