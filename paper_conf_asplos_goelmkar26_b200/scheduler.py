"""QoServe host scheduler (NEXT-1): builds each hybrid batch the engine executes.

Plain host code, written once and shared by the GPU runs and the oracle runs (BASELINE.json
north star).  It follows the paper's §3:

* QoS classes and deadlines (§3.2, Eq. 1-3): interactive requests carry
  TTFT + TBT SLOs, non-interactive ones a TTLT SLO;
      D_first = t_arr + SLO_TTFT
      D_n     = t_arr + SLO_TTFT + (n - 1) * SLO_TBT     (Eq. 2 is garbled; reading s17)
      D_total = t_arr + SLO_TTLT
* dynamic chunking (§3.3, §3.6.1): the prefill budget C is the
  largest chunk whose predicted step latency fits the minimum decode slack, slack = deadline of
  a decode's next token - now; the predictor is `latency_model.LatencyModel` fitted to the
  engine's own `qos_profile_step` table and biased to under-predict the chunk (margin);
* hybrid prioritisation (§3.4, Eq. 4-5):
      interactive:      P = t_arr + SLO_TTFT + alpha * Prefill_rem
      non-interactive:  P = t_arr + SLO_TTLT + alpha * (Prefill_rem + Decode_rem)
  with Decode_rem = per-application history mean + 2 sigma and
  alpha in ms/token (8 ms/token at fixed QPS);
* eager relegation with application hints (free tier first, PAPER.md:
  736-741, 923-926); relegated requests sort last and are served opportunistically;
* selective preemption: decodes are never preempted; a partially prefilled
  request is displaced only if waiting one more iteration does not make it violate;
* Algorithm 1 CREATE_BATCH / COMPARATOR.

Readings for the silent points: slack of a TTLT-only decode =
(D_total - now) / max(1, predicted remaining decodes); WILL_VIOLATE = now + predicted time to
finish the current phase > its deadline; relegation pops, marks and re-pushes the job (the
pseudo-code's lines 12-15 would otherwise spin).
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

# Table 3: QoS buckets, equal thirds
QOS_TIERS = {
    "Q1": {"interactive": True, "ttft": 6.0, "tbt": 0.050, "ttlt": None},
    "Q2": {"interactive": False, "ttft": None, "tbt": None, "ttlt": 600.0},
    "Q3": {"interactive": False, "ttft": None, "tbt": None, "ttlt": 1800.0},
}


@dataclass
class Request:
    req_id: int
    t_arrival: float
    prompt_len: int
    tier: str
    app_id: str = "default"
    important: bool = True            # application hint (paid vs free tier)
    decode_len: int = 1               # ground truth, known to the replay, never to the scheduler
    # state
    prefill_done: int = 0
    decoded: int = 0                  # output tokens produced (the first comes with the prefill)
    relegated: bool = False
    t_first: float | None = None
    t_last: float | None = None
    token_times: list = field(default_factory=list)

    @property
    def qos(self) -> dict:
        return QOS_TIERS[self.tier]

    @property
    def interactive(self) -> bool:
        return self.qos["interactive"]

    @property
    def prefill_rem(self) -> int:
        return self.prompt_len - self.prefill_done

    @property
    def ctx_len(self) -> int:
        """Tokens in the KV cache while decoding: the prompt plus the tokens fed back so far."""
        return self.prompt_len + self.decoded - 1

    # ---------------------------------------------------------------- deadlines (Eq. 1-3)
    def d_first(self) -> float:
        return self.t_arrival + self.qos["ttft"]

    def d_token(self, n: int) -> float:
        """Deadline of the n-th output token (n = 1 is the first), Eq. 2."""
        return self.t_arrival + self.qos["ttft"] + (n - 1) * self.qos["tbt"]

    def d_total(self) -> float:
        return self.t_arrival + self.qos["ttlt"]

    def done(self) -> bool:
        return self.decoded >= self.decode_len


class DecodeHistory:
    """Per-application decode-length history; the estimate is mean + 2 sigma."""

    def __init__(self, default: float = 128.0):
        self.default = default
        self.stats: dict[str, list] = {}

    def observe(self, app: str, n: int) -> None:
        s = self.stats.setdefault(app, [0, 0.0, 0.0])
        s[0] += 1
        s[1] += n
        s[2] += n * n

    def estimate(self, app: str) -> float:
        s = self.stats.get(app)
        if not s or s[0] < 2:
            return self.default
        mean = s[1] / s[0]
        var = max(0.0, s[2] / s[0] - mean * mean)
        return mean + 2.0 * math.sqrt(var)


@dataclass
class SchedulerConfig:
    alpha_ms_per_token: float = 8.0
    max_chunk: int = 4096             # throughput saturates (Fig. 4 analogue)
    min_chunk: int = 64
    chunk_step: int = 64
    margin: float = 0.05              # under-predict the chunk
    max_decodes: int = 256
    max_rows: int = 264               # engine capacity: chunks + decodes per step (max_batch_rows)
    max_tokens: int | None = None     # engine capacity: prefill tokens + decodes per step
                                      # (max_batch_tokens); None = unbounded
    # "slack": QoServe's dynamic chunking (the chunk fits the minimum decode slack);
    # "medha": Medha-style adaptive chunking (NEXT-4 variant): every step
    # targets a fixed latency, so chunks shrink as the prefill's cached prefix grows
    chunk_policy: str = "slack"
    medha_target_ms: float = 50.0
    # ablation switches (the paper's Medha comparison runs "only dynamic chunking under FCFS
    # scheduling, disabling all other techniques"): fcfs orders the prefill
    # queue by arrival instead of the hybrid priority; relegation / preemption toggle eager
    # relegation (Alg. 1 lines 12-15) and selective preemption
    fcfs: bool = False
    relegation: bool = True
    preemption: bool = True


class QoServeScheduler:
    def __init__(self, cfg: SchedulerConfig, predict_ms, history: DecodeHistory | None = None):
        """predict_ms(chunks=[(kv_start, len)], ctx=[...]) -> predicted step latency (ms)."""
        self.cfg = cfg
        self.predict_ms = predict_ms
        self.history = history or DecodeHistory()
        self.prefill_q: list[Request] = []   # includes relegated requests (they sort last)
        self.decode_q: list[Request] = []

    # ---------------------------------------------------------------- bookkeeping
    def submit(self, r: Request) -> None:
        self.prefill_q.append(r)

    def priority(self, r: Request) -> float:
        """Hybrid priority, Eq. 4 / Eq. 5 (seconds; alpha in ms/token)."""
        a = self.cfg.alpha_ms_per_token * 1e-3
        if r.interactive:
            return r.t_arrival + r.qos["ttft"] + a * r.prefill_rem
        decode_rem = max(0.0, self.history.estimate(r.app_id) - r.decoded)
        return r.t_arrival + r.qos["ttlt"] + a * (r.prefill_rem + decode_rem)

    def sort_key(self, r: Request):
        """COMPARATOR (Alg. 1 lines 26-33): non-relegated first, then priority (fcfs: arrival)."""
        if self.cfg.fcfs:
            return (r.relegated, r.t_arrival, r.req_id)
        return (r.relegated, self.priority(r), r.t_arrival, r.req_id)

    # ---------------------------------------------------------------- slack / budget
    def next_token_deadline(self, r: Request) -> float:
        if r.interactive:
            return r.d_token(r.decoded + 1)
        return r.d_total()

    def slack(self, r: Request, now: float) -> float:
        if r.interactive:
            return self.next_token_deadline(r) - now
        rem = max(1.0, self.history.estimate(r.app_id) - r.decoded)
        return (r.d_total() - now) / rem        # reading s19

    def min_slack(self, now: float) -> float:
        return min((self.slack(r, now) for r in self.decode_q), default=math.inf)

    def prefill_budget(self, ctx: list, min_slack_s: float, kv_start: int = 0) -> int:
        """GET_PREFILL_BUDGET (Alg. 1 line 7): largest chunk with predicted latency within the
        minimum decode slack (with margin); max_chunk when no decode constrains the step.  The
        prediction prices the chunk at `kv_start` (the cached prefix of the request it will
        come from: attention over the prefix grows for later chunks).
        Medha policy: the budget is a fixed per-step latency target instead of the slack."""
        if self.cfg.chunk_policy == "medha":
            budget_ms = self.cfg.medha_target_ms * (1 - self.cfg.margin)
            if math.isfinite(min_slack_s):
                budget_ms = min(budget_ms, max(0.0, min_slack_s) * 1e3 * (1 - self.cfg.margin))
        elif not math.isfinite(min_slack_s):
            return self.cfg.max_chunk
        else:
            budget_ms = max(0.0, min_slack_s) * 1e3 * (1 - self.cfg.margin)
        best = 0
        c = self.cfg.min_chunk
        while c <= self.cfg.max_chunk:
            if self.predict_ms([(kv_start, c)], ctx) <= budget_ms:
                best = c
            else:
                break
            c += self.cfg.chunk_step
        return best

    def step_estimate_s(self, chunk: int, ctx: list, kv_start: int = 0) -> float:
        return self.predict_ms([(kv_start, chunk)] if chunk else [], ctx) * 1e-3

    def will_violate(self, r: Request, now: float, chunk: int, ctx: list) -> bool:
        """now + predicted time to finish the current phase > deadline (reading s19)."""
        if chunk <= 0:
            return False
        steps = math.ceil(r.prefill_rem / chunk)
        t_done = now + steps * self.step_estimate_s(chunk, ctx)
        if r.interactive:
            return t_done > r.d_first()
        dec = max(0.0, self.history.estimate(r.app_id) - r.decoded)
        return t_done + dec * self.step_estimate_s(0, ctx or [r.prompt_len]) > r.d_total()

    # ---------------------------------------------------------------- Algorithm 1
    def create_batch(self, now: float):
        """Returns (chunks [(Request, n_tokens)], decodes [Request]).

        Capacity (the engine's, not the paper's): a chunk that completes its request's prefill
        turns it into a decode at the end of the step, so such chunks are only taken while
        decodes + finishing prefills stay within max_decodes; a chunk that would overflow the
        decode set is cut one token short of the prompt's end (it keeps progressing and finishes
        once a decode slot frees).  The decode set therefore never exceeds max_decodes and every
        decode is scheduled every step (decodes are never preempted)."""
        decodes = list(self.decode_q)[: self.cfg.max_decodes]          # GET_ALL_DECODES
        ctx = [r.ctx_len for r in decodes]                              # GET_DECODE_CONTEXT
        queue = sorted(self.prefill_q, key=self.sort_key)               # line 8
        kv0 = queue[0].prefill_done if queue else 0                     # prefix of the head chunk
        C = self.prefill_budget(ctx, self.min_slack(now), kv0)          # lines 5-7
        if self.cfg.max_tokens is not None:
            C = max(0, min(C, self.cfg.max_tokens - len(decodes)))
        chunks, count = [], 0
        finishing = 0                     # chunks of this batch that complete their prefill

        def fit(r: Request, want: int) -> int:
            """Tokens of r to take: want, unless that finishes r into a full decode set."""
            if want >= r.prefill_rem and len(self.decode_q) + finishing >= self.cfg.max_decodes:
                return r.prefill_rem - 1
            return want

        i = 0
        while count < C and i < len(queue) and len(chunks) + len(decodes) < self.cfg.max_rows:   # line 10
            top = queue[i]
            if top.prefill_done == 0 and len(self.decode_q) + finishing >= self.cfg.max_decodes:
                # admission: a new prompt is not started while the decode set is full
                i += 1
                continue
            if self.cfg.relegation and not top.relegated and self.will_violate(top, now, C, ctx):   # line 12
                # eager relegation with hints: free-tier first; important requests only once
                # they have actually missed their deadline
                deadline = top.d_first() if top.interactive else top.d_total()
                if not top.important or now > deadline:
                    top.relegated = True                                # lines 13-14
                    queue.append(queue.pop(i))                          # re-pushed, sorts last
                    continue
            take = fit(top, min(C - count, top.prefill_rem))            # line 17
            if take > 0:
                chunks.append((top, take))                              # lines 18-20
                count += take
                finishing += take == top.prefill_rem
            i += 1                                                      # line 21 (POP)
        # selective preemption: an already started prefill that was displaced keeps its slot
        # when waiting one more iteration would make it violate -- but only
        # within what is left of the budget C (the decode slack bounds the whole step)
        chosen = {r.req_id for r, _ in chunks}
        for r in (queue[i:] if self.cfg.preemption else []):
            if count >= C or len(chunks) + len(decodes) >= self.cfg.max_rows:
                break
            if r.prefill_done > 0 and r.req_id not in chosen and not r.relegated:
                if self.will_violate(r, now + self.step_estimate_s(C, ctx), max(C, 1), ctx):
                    take = fit(r, min(C - count, r.prefill_rem))
                    if take > 0:
                        chunks.append((r, take))
                        count += take
                        finishing += take == r.prefill_rem
        return chunks, decodes

    def complete(self, chunks, decodes, t_end: float) -> list[Request]:
        """Account one executed step ending at t_end; returns the finished requests."""
        finished = []
        for r, n in chunks:
            r.prefill_done += n
            if r.prefill_rem == 0:                # prefill done -> first token (step 7, Fig. 3)
                self.prefill_q.remove(r)
                r.decoded = 1
                r.t_first = t_end
                r.token_times.append(t_end)
                if r.done():
                    r.t_last = t_end
                    finished.append(r)
                else:
                    self.decode_q.append(r)
        for r in decodes:
            r.decoded += 1
            r.token_times.append(t_end)
            if r.done():
                r.t_last = t_end
                self.decode_q.remove(r)
                finished.append(r)
        for r in finished:
            self.history.observe(r.app_id, r.decode_len)
        return finished


def violated(r: Request) -> bool:
    """SLO check of a finished request: TTFT and every TBT deadline (interactive) or TTLT."""
    if r.t_last is None:
        return True
    if r.interactive:
        if r.t_first > r.d_first():
            return True
        return any(t > r.d_token(n + 1) for n, t in enumerate(r.token_times))
    return r.t_last > r.d_total()
