"""Online serving loop: the scheduler (include/tcb.h §5) feeding the B200 encoder.

TCB's service model (§3, §5.1): requests arrive over time, and whenever
the GPU is idle the scheduler turns the waiting set into one batch of B rows x L words.
The batch runs through the ConcatBatching encoder and its responses are returned.  Here:

* the request stream (arrival, deadline, length, token ids) is given up front; requests
  are submitted to the C++ scheduler when the clock passes their arrival;
* each time slot: ``tcb_sched_next_batch(now)`` -> plan of exactly B rows -> its segment
  table and token ids are copied into fixed device buffers -> one CUDA-graph replay of
  forward + unpack (the graph is captured once: the kernels read only the device segment
  table, include/tcb.h §1) -> the stream is synchronised (the GPU is idle again);
* the clock advances by the scheduler's host time (measured around the C++ call) plus the
  batch's device time (CUDA events around H2D + graph), so utility and throughput are those
  of a serial scheduler + GPU pipeline on this hardware.  When no request is waiting, the
  clock jumps to the next arrival.
* ``overlap=True``: a two-deep pipeline.  Right after batch k is enqueued (slot start S_k),
  the host schedules batch k+1 from the requests that arrived by S_k, with deadlines checked
  against its predicted start S_k + (mean device time so far), and enqueues it behind batch k
  (double-buffered device segment table / ids / responses, one captured graph per buffer).
  Batch k+1 starts at S_{k+1} = S_k + max(device time of k, scheduling time of k+1): the
  scheduler's host time hides behind the GPU (the paper's overhead argument, P:1805-1811,
  without the serial sum), at the price of not seeing arrivals during batch k until slot k+2.

All compute runs in libtcb's kernels; this module only moves buffers and keeps time.
"""
from __future__ import annotations

import time
from typing import Dict

import numpy as np

from . import Encoder, Scheduler


class Server:
    def __init__(self, encoder: Encoder, policy: str, batch_rows: int, row_len: int,
                 eta: float = 0.5, q: float = 0.5, overlap: bool = False):
        import torch
        self.overlap = bool(overlap)
        self.enc = encoder
        self.B, self.L = int(batch_rows), int(row_len)
        self.policy, self.eta, self.q = policy, eta, q
        M = self.B * self.L
        d = encoder.model.d_model
        dev = encoder.device
        # segment table of at most M segments (one per slot) + row index + query-block order
        self.seg_words = 4 * (1 + M) + ((self.B + 1 + 3) // 4) * 4 + ((M + 127) // 128 + 3) // 4 * 4
        self.d_segtab = torch.zeros(self.seg_words, dtype=torch.int32, device=dev)
        self.h_segtab = torch.zeros(self.seg_words, dtype=torch.int32).pin_memory()
        self.d_ids = torch.zeros(M, dtype=torch.int32, device=dev)
        self.h_ids = torch.zeros(M, dtype=torch.int32).pin_memory()
        self.rows = encoder.alloc_rows(M)
        self.out = torch.zeros((M, d), dtype=encoder.dtype, device=dev)
        self.stream = torch.cuda.Stream()
        self.graph = None
        self.last_batch = None
        self.last_out = self.out
        if self.overlap:   # second set of per-batch buffers (slot 1; slot 0 is the above)
            self.bufs = [(self.d_segtab, self.d_ids, self.out, self.h_segtab, self.h_ids),
                         (torch.zeros_like(self.d_segtab), torch.zeros_like(self.d_ids),
                          torch.zeros_like(self.out),
                          torch.zeros(self.seg_words, dtype=torch.int32).pin_memory(),
                          torch.zeros(M, dtype=torch.int32).pin_memory())]
            self.graphs = [None, None]

    def _capture(self, plan) -> None:
        import torch
        s = self.stream
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s):
            for _ in range(2):
                self.enc.encoder_forward_unpacked(plan, self.d_segtab, self.d_ids, self.out, self.rows, stream=s)
        s.synchronize()
        self.graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(self.graph, stream=s):
            self.enc.encoder_forward_unpacked(plan, self.d_segtab, self.d_ids, self.out, self.rows, stream=s)

    def _capture_slot(self, k, plan) -> None:
        import torch
        d_seg, d_ids, out = self.bufs[k][:3]
        s = self.stream
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s):
            for _ in range(2):
                self.enc.encoder_forward_unpacked(plan, d_seg, d_ids, out, self.rows, stream=s)
        s.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            self.enc.encoder_forward_unpacked(plan, d_seg, d_ids, out, self.rows, stream=s)
        self.graphs[k] = g

    def _run_overlap(self, lengths, arrival, deadline, token_ids, tok_offsets, horizon):
        import torch
        n = len(lengths)
        sched = Scheduler(self.policy, self.B, self.L, self.eta, self.q)
        order = np.argsort(arrival, kind="stable")
        arr_sorted = arrival[order]
        nxt = 0
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
              for _ in range(2)]
        batches, gpu_ms, sched_ms, tokens = 0, 0.0, 0.0, 0
        now = 0.0                 # start of the batch in flight (or the host clock when idle)
        inflight = None           # (slot, ids, lens)
        k = 0                     # buffer slot of the next batch

        def finish(slot_ids_lens):
            nonlocal gpu_ms, batches, tokens
            kp, ids_p, lens_p = slot_ids_lens
            ev[kp][1].synchronize()
            g = ev[kp][0].elapsed_time(ev[kp][1])
            gpu_ms += g
            batches += 1
            tokens += int(lens_p.sum())
            self.last_batch, self.last_out = (ids_p, lens_p), self.bufs[kp][2]
            return g / 1e3

        while now <= horizon:
            end = int(np.searchsorted(arr_sorted, now, side="right"))
            if end > nxt:                          # arrivals up to the current slot start
                sel = order[nxt:end]
                sched.submit(sel, lengths[sel], arrival[sel], deadline[sel])
                nxt = end
            est = (gpu_ms / batches / 1e3) if batches else 0.0
            t0 = time.perf_counter()
            ids, lens, plan = sched.next_batch(now + (est if inflight is not None else 0.0))
            t_sched = time.perf_counter() - t0
            sched_ms += t_sched * 1e3
            if len(ids) > 0:
                d_seg, d_ids, out, h_seg, h_ids = self.bufs[k]
                words = plan.segtab()
                h_seg[:len(words)].copy_(torch.from_numpy(words))
                tok = np.concatenate([token_ids[tok_offsets[i]:tok_offsets[i] + lengths[i]]
                                      for i in ids])
                h_ids[:len(tok)].copy_(torch.from_numpy(tok))
                if self.graphs[k] is None:         # first use of this buffer slot
                    self.stream.synchronize()
                    d_seg.copy_(h_seg)
                    self._capture_slot(k, plan)
                with torch.cuda.stream(self.stream):
                    ev[k][0].record(self.stream)
                    d_seg.copy_(h_seg, non_blocking=True)
                    d_ids[:len(tok)].copy_(h_ids[:len(tok)], non_blocking=True)
                    self.graphs[k].replay()
                    ev[k][1].record(self.stream)
            # the batch in flight completes; the new one starts once both it and the new
            # one's scheduling are done
            if inflight is not None:
                now += max(finish(inflight), t_sched)
            else:
                now += t_sched
            if len(ids) > 0:
                inflight = (k, ids, lens)
                k ^= 1
            else:
                inflight = None
                if sched.stats()["waiting"] == 0:
                    if nxt >= n:
                        break
                    now = max(now, float(arr_sorted[nxt]))
        if inflight is not None:
            now += finish(inflight)
        return self._result(sched, n, now, tokens, batches, gpu_ms, sched_ms)

    def _result(self, sched, n, now, tokens, batches, gpu_ms, sched_ms):
        st = sched.stats()
        elapsed = max(now, 1e-12)
        return {"policy": self.policy, "B": self.B, "L": self.L, "requests": n,
                "overlap": self.overlap, "tokens": tokens,
                "scheduled": st["scheduled"], "expired": st["expired"],
                "utility": st["utility"], "sim_seconds": elapsed,
                "responses_per_s": st["scheduled"] / elapsed,
                "tokens_per_s": tokens / elapsed, "batches": batches,
                "batch_ms": gpu_ms / max(batches, 1),
                "sched_ms": sched_ms / max(st["batches"], 1),
                "sched_over_batch": (sched_ms / max(st["batches"], 1)) /
                                    max(gpu_ms / max(batches, 1), 1e-12)}

    def run(self, lengths, arrival, deadline, token_ids, tok_offsets,
            horizon: float) -> Dict[str, float]:
        """Serve the stream until the clock passes ``horizon`` seconds (or the stream is
        exhausted).  Returns utility / throughput / timing statistics."""
        import torch
        if self.overlap:
            return self._run_overlap(lengths, arrival, deadline, token_ids, tok_offsets, horizon)

        n = len(lengths)
        sched = Scheduler(self.policy, self.B, self.L, self.eta, self.q)
        order = np.argsort(arrival, kind="stable")
        arr_sorted = arrival[order]
        nxt = 0                                    # next request (in arrival order) to submit
        now = 0.0
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        batches, gpu_ms, sched_ms, tokens = 0, 0.0, 0.0, 0
        while now <= horizon:
            end = int(np.searchsorted(arr_sorted, now, side="right"))
            if end > nxt:                          # arrivals up to now
                sel = order[nxt:end]
                sched.submit(sel, lengths[sel], arrival[sel], deadline[sel])
                nxt = end
            t0 = time.perf_counter()
            ids, lens, plan = sched.next_batch(now)
            t_sched = time.perf_counter() - t0
            sched_ms += t_sched * 1e3
            if len(ids) == 0:
                if nxt >= n:
                    break
                now = max(now + t_sched, float(arr_sorted[nxt]))
                continue
            words = plan.segtab()
            self.h_segtab[:len(words)].copy_(torch.from_numpy(words))
            tok = np.concatenate([token_ids[tok_offsets[i]:tok_offsets[i] + lengths[i]] for i in ids])
            self.h_ids[:len(tok)].copy_(torch.from_numpy(tok))
            if self.graph is None:
                self.d_segtab.copy_(self.h_segtab)
                self._capture(plan)
            with torch.cuda.stream(self.stream):
                ev0.record(self.stream)
                self.d_segtab.copy_(self.h_segtab, non_blocking=True)
                self.d_ids[:len(tok)].copy_(self.h_ids[:len(tok)], non_blocking=True)
                self.graph.replay()
                ev1.record(self.stream)
            self.stream.synchronize()
            g = ev0.elapsed_time(ev1)
            self.last_batch = (ids, lens)        # its responses are in self.out[:sum(lens)]
            self.last_out = self.out
            gpu_ms += g
            batches += 1
            tokens += int(lens.sum())
            now += t_sched + g / 1e3
        return self._result(sched, n, now, tokens, batches, gpu_ms, sched_ms)
