"""Sequential-task-flow (STF) DAG recorder.

Input generator only: it holds none of the MultiPrio arithmetic (scores,
bottom-levels, queues).  It reproduces how the runtime infers the DAG from the
data-access modes and the submission order (§I, l.91 §III-A:
"the runtime system infers the DAG automatically by taking into account the
data dependencies between tasks"), at handle granularity:

* RAW / WAW: the last writer of a handle precedes every later reader/writer;
* WAR: every reader since the last write precedes the next writer.

Edges are emitted raw, duplicates included (a task reading two handles last
written by the same predecessor produces two identical edges), exactly as a
runtime would observe them; deduplication is step a1 of the hot path
(SURVEY.md §8(c) reading c19).
"""
from __future__ import annotations

import numpy as np


class STFRecorder:
    __slots__ = ("n", "kind", "_src", "_dst", "_last_writer", "_readers", "_acc_h", "_acc_m", "_acc_ptr")

    def __init__(self) -> None:
        self.n = 0
        self.kind: list[int] = []
        self._src: list[int] = []
        self._dst: list[int] = []
        self._last_writer: dict = {}
        self._readers: dict = {}
        self._acc_h: list[int] = []        # data accesses of every task
        self._acc_m: list[int] = []        # 1 = R, 3 = RW
        self._acc_ptr: list[int] = [0]

    def submit(self, kind: int, reads=(), writes=()) -> int:
        """Submit one task.  `reads` are R handles, `writes` are RW handles."""
        t = self.n
        self.n += 1
        self.kind.append(kind)
        lw_map = self._last_writer
        rd_map = self._readers
        src = self._src
        dst = self._dst
        for h in reads:
            self._acc_h.append(h)
            self._acc_m.append(1)
            lw = lw_map.get(h)
            if lw is not None:
                src.append(lw)
                dst.append(t)
            lst = rd_map.get(h)
            if lst is None:
                rd_map[h] = [t]
            else:
                lst.append(t)
        for h in writes:
            self._acc_h.append(h)
            self._acc_m.append(3)
            lw = lw_map.get(h)
            if lw is not None:
                src.append(lw)
                dst.append(t)
            lst = rd_map.get(h)
            if lst:
                for r in lst:
                    if r != t:
                        src.append(r)
                        dst.append(t)
                rd_map[h] = []
            lw_map[h] = t
        self._acc_ptr.append(len(self._acc_h))
        return t

    def edges(self) -> tuple[np.ndarray, np.ndarray]:
        return (np.asarray(self._src, dtype=np.int32),
                np.asarray(self._dst, dtype=np.int32))

    def kinds(self) -> np.ndarray:
        return np.asarray(self.kind, dtype=np.int32)

    def accesses(self) -> tuple[np.ndarray, np.ndarray, np.ndarray]:
        """(acc_ptr int64[n+1], handle int32[acc], mode uint8[acc]; 1 = R, 3 = RW).
        Handle keys are renumbered densely 0..H-1 in increasing key order."""
        h = np.asarray(self._acc_h, dtype=np.int64)
        if len(h) and (h.min() < 0 or h.max() >= len(h)):
            _, h = np.unique(h, return_inverse=True)
        return (np.asarray(self._acc_ptr, dtype=np.int64), h.astype(np.int32),
                np.asarray(self._acc_m, dtype=np.uint8))
