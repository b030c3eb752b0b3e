"""fp64 CPU oracle for the Astra custom-RNN training step — TEST INFRASTRUCTURE ONLY.

Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s `cpu_baseline` / `--impl reference`
legs may import anything from here.  The product path (the C-ABI library under
`paper_conf_asplos_sivathanucsz19_b200/`) never imports, links or calls this package, and this
package imports nothing from the product path: the two share no code, headers, tables or
helpers.  The only thing both sides see is the seeded input generator module `synth/`.

What it computes (§6.7): Astra's optimisations are *value-preserving*, so the
result of an optimised training step is exactly the plain definition of the step.  The
oracle is that definition written out in fp64 numpy with explicit per-timestep loops and a
hand-derived backward (no autograd):

* `cells`  — forward + backward through time of LSTM, MI-LSTM [36], SC-RNN [22], RHN [39],
             subLSTM [8] and the reduced LSTM-with-attention [35];
* `lm`     — embedding, LM head, mean cross-entropy, SGD, one full LM training step;
* `dp`     — data-parallel semantics (mean of shard gradients);
* `tuner`  — the exploration semantics of the update tree / profile index on an
             injected cost table.

The paper prints no cell equations (only citations) and no worked numeric example; every
reading taken is listed in DESIGN.md "Readings of the paper".  Pins (tests/test_oracle_*.py):
reductions to torch.nn.LSTM / torch.nn.RNN in fp64, closed forms, central finite
differences, statefulness, DP linearity, and the paper's worked exploration counts.
"""
