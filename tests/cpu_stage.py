"""CPU stand-in for one rank's device stage of the sharded check -- TEST INFRASTRUCTURE.

Implements the stage interface of paper_conf_sosp_kamathb21_b200.dist (prepare / detect) with
numpy and the CPU oracle, so the distributed orchestration (chunking, owner routing, all-to-all,
all-gather, reductions, merge) can be exercised with torch.distributed/gloo on CPU.  detect()
rebuilds the rank's shard trace -- the global synchronization stream plus the received accesses,
in global order -- runs the oracle on it and keeps the reports on the words the rank owns (whose
histories are complete there)."""
import numpy as np
import torch

import oracle
import tracegen as tg
from paper_conf_sosp_kamathb21_b200.dist import NONE64, owner_of


class CpuStage:
    def load(self, chunk, first_event, n_total, n_blocks, block_dim):
        self.ev = np.ascontiguousarray(chunk)
        self.first, self.n_total, self.nb, self.bd = first_event, n_total, n_blocks, block_dim

    def prepare(self, nranks):
        self.P = nranks
        addr, tid, kind, scope, mask = tg.unpack(self.ev)
        gidx = np.arange(len(self.ev), dtype=np.int64) + self.first
        acc = kind <= 4
        words = (addr >> np.uint64(2))
        own = owner_of(words[acc], nranks)
        recs = np.stack([(words[acc] & np.uint64(0xFFFFFFFF)).astype(np.uint32).view(np.int32),
                         gidx[acc].astype(np.uint32).view(np.int32), self.ev["tk"][acc].view(np.int32),
                         mask[acc].view(np.int32)], axis=1) if acc.any() else np.zeros((0, 4), np.int32)
        order = np.argsort(own, kind="stable")
        counts = np.bincount(own, minlength=nranks).tolist() if acc.any() else [0] * nranks
        sync = (kind >= 5) | (kind == 3) | (kind == 4)
        sev = self.ev[sync].view(np.int32).reshape(-1, 4) if sync.any() else np.zeros((0, 4), np.int32)
        wmin = int(words[acc].min()) if acc.any() else NONE64
        wmax = int(words[acc].max()) if acc.any() else 0
        return {"records": torch.from_numpy(np.ascontiguousarray(recs[order])), "counts": counts,
                "sync_idx": torch.from_numpy(gidx[sync].astype(np.int32)),
                "sync_ev": torch.from_numpy(np.ascontiguousarray(sev)), "bad": NONE64, "min_word": wmin,
                "max_word": wmax}

    def detect(self, recv, sync_idx, sync_ev, min_word, timing=False, paper_counters=False):
        me = getattr(self, "rank", None)
        recv = recv.numpy()
        sidx = sync_idx.numpy().astype(np.uint32).astype(np.int64)
        sev = np.ascontiguousarray(sync_ev.numpy()).view(tg.EVENT_DTYPE).reshape(-1)
        key = recv[:, 0].view(np.uint32).astype(np.uint64)
        word = np.uint64(min_word) + ((key - np.uint64(min_word & 0xFFFFFFFF)) & np.uint64(0xFFFFFFFF))
        racc = np.zeros(len(recv), tg.EVENT_DTYPE)
        racc["addr"] = word << np.uint64(2)
        racc["tk"] = recv[:, 2].view(np.uint32)
        racc["mask"] = recv[:, 3].view(np.uint32)
        ridx = recv[:, 1].view(np.uint32).astype(np.int64)
        # union by global index (an owned CAS/EXCH is in both streams)
        allidx = np.concatenate([sidx, ridx])
        allev = np.concatenate([sev, racc])
        uniq, first = np.unique(allidx, return_index=True)
        trace = allev[first]
        rep = oracle.run(trace, self.nb, self.bd, paper_counters=paper_counters)
        mine = owner_of(rep["addr"] >> np.uint64(2), self.P) == self.rank
        rep = rep[mine].copy()
        rep["cur"] = uniq[rep["cur"].astype(np.int64)]
        rep["prev"] = uniq[rep["prev"].astype(np.int64)]
        return rep
