"""Pins of the context-switch oracle (oracle/switch_model.py).

PAPER.md:575-598 -- each EST must behave exactly like a dedicated DDP worker:
its RNG and BatchNorm state evolve only through its own local steps, however
the ESTs are interleaved on one GPU.  The pin is that definition written as
N independent workers: any interleaving of (switch, update) events applied to
the time-sliced model must leave every EST with the state of its dedicated
worker."""
import numpy as np

from oracle.switch_model import SwitchModel


def test_switch_model_equals_dedicated_workers():
    rng = np.random.default_rng(0)
    for trial in range(50):
        N = int(rng.integers(1, 9))
        sizes = [16, int(rng.integers(1, 64))]
        init = {k: [rng.integers(0, 256, s, dtype=np.uint8).tobytes() for s in sizes] for k in range(N)}
        dedicated = {k: list(init[k]) for k in range(N)}      # one worker per EST, never switching
        m = SwitchModel(N, init)
        cur = 0
        for _ in range(100):
            if rng.random() < 0.5:
                cur = int(rng.integers(0, N))
                m.switch(cur)
            else:
                i = int(rng.integers(0, len(sizes)))
                nb = rng.integers(0, 256, sizes[i], dtype=np.uint8).tobytes()
                m.mutate(i, nb)                  # the running EST updates its own state ...
                dedicated[cur][i] = nb           # ... exactly as its dedicated worker would
        for k in range(N):
            assert m.state_of(k) == dedicated[k]


def test_switch_to_self_and_round_trip():
    init = {0: [b"a" * 16], 1: [b"b" * 16]}
    m = SwitchModel(2, init)
    m.switch(0)
    assert m.state_of(0) == [b"a" * 16]
    m.mutate(0, b"c" * 16)
    m.switch(1)
    m.switch(0)
    assert m.state_of(0) == [b"c" * 16] and m.state_of(1) == [b"b" * 16]
