"""Context-switch oracle: a dictionary state machine.  TEST INFRASTRUCTURE ONLY.

PAPER.md:575-598 -- an EST's context is what cannot be shared between the ESTs
time-sliced on one worker: RNG states, implicit
per-worker framework state such as BatchNorm running statistics,
and gradients (handled by the stash).  Parameters and optimizer state are one
shared replica.

Model: one "live" copy of each registered state buffer (what the running EST
reads and writes), and one saved copy per EST.  ``switch(k)`` saves live into
cur's saved copy, then loads k's saved copy into live, and sets cur = k.

Correctness criterion (pinned in tests): after any interleaving of switches
and state mutations, each EST's state equals what a *dedicated* worker (one
EST per GPU, never switching) would hold after the same per-EST mutations.
"""


class SwitchModel:
    def __init__(self, n_est, initial):
        """initial: dict est -> list of bytes (one entry per registered buffer)."""
        self.n = n_est
        self.saved = {k: [bytes(b) for b in initial[k]] for k in range(n_est)}
        self.cur = 0
        self.live = [bytes(b) for b in self.saved[0]]

    def switch(self, k):
        if not (0 <= k < self.n):
            raise ValueError("bad est")
        self.saved[self.cur] = list(self.live)        # save the outgoing EST
        self.live = list(self.saved[k])               # load the incoming one
        self.cur = k

    def mutate(self, idx, new_bytes):
        """The running EST changes live buffer idx (e.g. BN update, RNG advance)."""
        assert len(new_bytes) == len(self.live[idx])
        self.live[idx] = bytes(new_bytes)

    def state_of(self, k):
        return list(self.live) if k == self.cur else list(self.saved[k])
