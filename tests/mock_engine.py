"""A CPU stand-in for libcuts behind dist.WorkSharing's engine interface.

It walks a synthetic search tree with the library's donation semantics
(include/cuts.h, cuts_set_donation / cuts_set_prefixes): levels are processed
depth-first in windows; at every window boundary ``poll(depth, remaining)`` is
asked about the shallowest level with unstarted entries, and donated entries
(the tail of that level) are shipped as flat prefix rows and never processed
here.  The tree is a deterministic function of the prefix, so the number of
leaves is known exactly.  Test infrastructure only.
"""
import time

import torch


def n_children(prefix, k):
    h = 1469598103934665603
    for x in prefix:
        h = ((h ^ (x + 1)) * 1099511628211) & 0xFFFFFFFFFFFFFFFF
    if prefix[0] == 0:
        return 16                       # one hub root: most of the work
    return (h >> 17) % 4


class MockEngine:
    def __init__(self, k=4, roots=40, window=2, delay=0.0005):
        self.k, self.roots, self.window, self.delay = k, roots, window, delay
        self.poll = self.ship = None
        self.processed_leaves = 0

    def set_hooks(self, poll, ship):
        self.poll, self.ship = poll, ship

    def serial_total(self):
        return self._levels([(r,) for r in range(self.roots)], 1, donate=False)

    def count_roots(self, b, e):
        return self._levels([(r,) for r in range(b, min(e, self.roots))], 1)

    def count_prefixes(self, rows):
        return self._levels([tuple(int(x) for x in row) for row in rows.tolist()], rows.shape[1])

    def _levels(self, entries, depth, donate=True):
        self.stack = {}
        return self._level(entries, depth, donate)

    def _maybe_donate(self):
        if not self.poll:
            return
        for d in sorted(self.stack):
            ents, nxt, end = self.stack[d]
            if end - nxt >= 2:
                give = min(int(self.poll(d, end - nxt)), end - nxt)
                if give > 0:
                    rows = torch.tensor(ents[end - give:end], dtype=torch.int32).reshape(give, d)
                    self.ship(d, rows)
                    self.stack[d][2] = end - give
                return

    def _level(self, entries, depth, donate):
        if depth == self.k:
            self.processed_leaves += len(entries)
            return len(entries)
        self.stack[depth] = [entries, 0, len(entries)]
        total, w0 = 0, 0
        while True:
            if donate:
                self._maybe_donate()
            end = self.stack[depth][2]
            if w0 >= end:
                break
            w1 = min(end, w0 + self.window)
            self.stack[depth][1] = w1
            children = [p + (c,) for p in entries[w0:w1] for c in range(n_children(p, self.k))]
            time.sleep(self.delay)
            total += self._level(children, depth + 1, donate) if children else 0
            w0 = w1
        del self.stack[depth]
        return total
