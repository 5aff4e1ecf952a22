"""CPU fp64 oracle of the QoServe hybrid-batch forward step — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import anything in this package.  The product path
(``paper_conf_asplos_goelmkar26_b200`` + ``libqoserve.so``) never imports it, and this
package never imports the product: the two share no code.

What it computes (§2.1 "chunked prefills ... without pausing ongoing
decodes"; §3.3 "fused prefill-decode MLP"; §3.6.1
"modifying the chunk size at runtime incurs no additional cost"): a hybrid step is a
batching / paging / chunking *schedule*, so every output row equals the plain, unbatched,
unchunked causal forward of a decoder-only transformer at that position.  The oracle is
that plain definition written out in fp64 from the bf16-rounded synthetic weights:

* ``oracle.gen``     — the synthetic-weight / KV-fill generator,
                       implemented independently of the CUDA generator.
* ``oracle.model``   — RMSNorm, RoPE, causal softmax attention, SwiGLU MLP, LM head
                       (Llama/Qwen2 convention, reading s1-s3).
* ``oracle.kv``      — the paged-KV block allocator (lowest free index first, block 16,
                       all-or-nothing; reading s12).
* ``oracle.engine``  — ``OracleEngine``: replays the same alloc/free/step calls as the
                       C ABI and returns fp64 logits rows.

Parity pins (tests/test_oracle_*.py): brute-force attention, softmax rows sum to 1,
chunk-split invariance, decode == last row of full causal prefill, batch-composition
invariance, RoPE norm/relative-position/identity, GEMM vs numpy fp64, closed forms.
"""
