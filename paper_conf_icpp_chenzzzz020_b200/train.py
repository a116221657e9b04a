"""Secure training / inference driver over the C ABI (the API a user calls).

Roles (Fig. 1b, L55-L65; Fig. 3):
  client  encodes plaintext (fixed point, f = 13) and splits it into two additive shares
          (psml_encode + psml_share on the GPU, streams keyed by the call-id layout below);
  dealer  generates the step's triplets / MSB material (psml_model_deal) -- the offline phase;
  servers run the online step on the shares (psml_secure_train_step), both parties co-resident.

Call-id layout (R11; part of the bit-exact contract with the oracle):
  pair[63:56] | step[55:24] | layer[23:16] | op[15:8] | slot[7:0]
  op 7 = share; slot 0 = X, 1 = Y, 2 = initial master weight (step = 0xFFFFFFFF).
Data parallelism: one co-resident pair per GPU, each on its own rows;
the untruncated weight-gradient shares are summed across pairs with an all-reduce (uint64 ring
addition = int64 two's-complement addition), then every pair applies the same update.
"""
import torch

from . import psml
from .parallel import dp_update_shift, ring_allreduce_

# The fixed seeds are the REPRODUCIBLE configuration (tests against the oracle, benchmarks): anyone
# knowing them can regenerate every share and mask.  A deployment draws secret ones (fresh_seeds).
DATA_SEED = 0x50534D4C
SHARE_SEED = DATA_SEED + 1
DEALER_SEED = DATA_SEED + 2


def fresh_seeds():
    """(share_seed, dealer_seed) from the OS CSPRNG, for a deployment: the client's sharing seed
    and the dealer's seed are then secret (the ChaCha20 keys of DESIGN.md R1 / R23)."""
    import secrets
    return secrets.randbits(64), secrets.randbits(64)
OP_SHARE = 7
INIT_STEP = 0xFFFFFFFF
KINDS = {"linreg": psml.LINREG, "logreg": psml.LOGREG, "mlp": psml.MLP, "cnn": psml.CNN, "svm": psml.SVM,
         "rnn": psml.RNN}
RNN_SHAPE = dict(dims=[32, 64, 10], rnn_steps=16)   # D, H, C and T (R25; synth.RNN_*)
WD_SHIFT = {"svm": 16}   # weight decay lambda.eta = 2^-16 (R24)
# forward-weight fractional bits per layer (R21); None = frac_bits for every layer
FWD_BITS = {"cnn": [16, 20, 20]}


def call_id(pair, step, layer, op, slot=0):
    return ((pair & 0xFF) << 56) | ((step & 0xFFFFFFFF) << 24) | ((layer & 0xFF) << 16) \
        | ((op & 0xFF) << 8) | (slot & 0xFF)


class SecureTrainer:
    """One co-resident party pair on the current GPU, training `task` with batch `batch`."""

    def __init__(self, task, W_init, batch=128, pair_id=0, dims=None, backend=0,
                 frac_bits=13, master_frac_bits=27, lr_shift=14, compare="a2b", dealer_seed=DEALER_SEED,
                 deal_role=0, w_shares=None, mask_reuse=False, strong_pairs=0, share_seed=SHARE_SEED):
        self.task = task
        self.ctx = psml.Ctx(l=64, frac_bits=frac_bits, backend=backend)
        self.ring = self.ctx.ring
        self.master_ring = psml.Ring(64, master_frac_bits)
        self.pair_id = pair_id
        self.batch = batch
        self.share_seed = share_seed   # the client's sharing seed (secret in a deployment: fresh_seeds)
        # strong scaling (R28): strong_pairs pairs share one global batch of
        # strong_pairs * batch rows; this pair trains rows [pair_id * batch, (pair_id + 1) * batch)
        self.strong_pairs = strong_pairs
        rnn = RNN_SHAPE if task == "rnn" else {}
        self.model = psml.Model(self.ctx, KINDS[task], dims=dims or rnn.get("dims"), batch=batch, lr_shift=lr_shift,
                                rnn_steps=rnn.get("rnn_steps", 0),
                                master_frac_bits=master_frac_bits, dealer_seed=dealer_seed, deal_role=deal_role,
                                pair_id=pair_id, fwd_frac_bits=FWD_BITS.get(task),
                                compare={"a2b": 0, "fss": 1}[compare], weight_decay_shift=WD_SHIFT.get(task, 0),
                                mask_reuse=mask_reuse, strong_pairs=strong_pairs)
        for layer, W in enumerate(W_init):
            if w_shares is not None:   # shares handed over by the client: w_shares[layer] = (Wm_0, Wm_1)
                self.model.set_master(layer, w_shares[layer])
                continue
            w = psml.encode(self.master_ring, torch.as_tensor(W, dtype=torch.float64))
            Wm = psml.share(self.ring, self.share_seed, call_id(0, INIT_STEP, layer, OP_SHARE, 2), w)
            self.model.set_master(layer, Wm)
        self.out_dim = self.model.layer_shape(self.model.n_layers - 1)[1]

    def d_in(self):
        """Features per input row: CNN 3x32x32, RNN T x D, else the first layer's fan-in."""
        if self.task == "cnn":
            return 3 * 32 * 32
        if self.task == "rnn":
            return RNN_SHAPE["rnn_steps"] * RNN_SHAPE["dims"][0]
        return self.model.layer_shape(0)[0]

    # --- client side -----------------------------------------------------------------------
    def _client_share(self, X, Y, step, outX=None, outY=None):
        """Client encode + share of a minibatch into (outX, outY): X float64
        features, or uint8 pixels (x = q / 255, synth.batch_u8); Y float64 labels, or uint8 class
        indices of one-hot labels.  Both forms give bit-identical shares."""
        cx = call_id(self.pair_id, step, 0, OP_SHARE, 0)
        cy = call_id(self.pair_id, step, 0, OP_SHARE, 1)
        if torch.is_tensor(X) and X.dtype == torch.uint8:
            Xs = psml.encode_share_u8(self.ring, self.share_seed, cx, X if X.is_cuda else X.cuda(non_blocking=True),
                                      255.0, out=outX)
        else:
            Xs = psml.encode_share(self.ring, self.share_seed, cx, _dev64(X), out=outX)
        if torch.is_tensor(Y) and Y.dtype == torch.uint8:
            Ys = psml.encode_share_onehot(self.ring, self.share_seed, cy, Y if Y.is_cuda else Y.cuda(non_blocking=True),
                                          self.out_dim, out=outY)
        else:
            Ys = psml.encode_share(self.ring, self.share_seed, cy, _dev64(Y), out=outY)
        return Xs, Ys

    def share_batch(self, X, Y, step):
        """Encode + share one minibatch on the GPU (X, Y: float64 tensors, host or device; or the
        uint8 pixel / class-index form, see _client_share)."""
        return self._client_share(X, Y, step)

    # --- steps --------------------------------------------------------------------------------
    def capture(self, with_update=True, pipelined=True):
        """Capture deal + online step (+ update) into CUDA graph(s) on a side stream; the batch is
        shared into fixed buffers before each replay (graph_step).  pipelined: the dealer of the
        next step runs concurrently with the online phase of this one (double-buffered pools)."""
        d_in = self.d_in()
        self.Xbuf = psml.empty_pair((self.batch, d_in), 64)
        self.Ybuf = psml.empty_pair((self.batch, self.out_dim), 64)
        for t in self.Xbuf + self.Ybuf:
            t.zero_()
        self.gstream = torch.cuda.Stream()
        self.gstream.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(self.gstream):
            self.model.capture_step(self.Xbuf, self.Ybuf, with_deal=True, with_update=with_update,
                                    pipelined=pipelined, stream=self.gstream)
        torch.cuda.current_stream().wait_stream(self.gstream)
        self.graph_update = with_update
        self.pipelined = pipelined
        self._next_dealt = None

    def graph_kernel_nodes(self):
        return self.model.graph_nodes()

    def graph_step(self, X, Y, step):
        """Client encode + share into the captured buffers, then replay the captured step (float64
        device batches: one library call, psml_model_step_device)."""
        if self.pipelined and self._next_dealt != step:
            self.model.deal(step)          # prime the pipeline (first step or a jump in step ids)
        if (torch.is_tensor(X) and torch.is_tensor(Y) and X.is_cuda and Y.is_cuda and X.dtype == torch.float64
                and Y.dtype == torch.float64):
            self.model.step_device(X.contiguous(), Y.contiguous(), self.share_seed, step)
        else:
            self._client_share(X, Y, step, outX=self.Xbuf, outY=self.Ybuf)
            self.model.step_graph(step)
        self._next_dealt = step + 1

    def graph_step_host(self, q, y, step, yhat_host):
        """The end-to-end client call: host pixels q (uint8) and labels y (float64, or uint8 class
        indices) in, the captured step on the GPU, both prediction shares out to yhat_host (host
        uint64, 2 x batch x d_L) -- one library call (psml_model_step_host), asynchronous."""
        if self.pipelined and self._next_dealt != step:
            self.model.deal(step)
        self.model.step_host(q, y, self.share_seed, step, yhat_host)
        self._next_dealt = step + 1

    def deal(self, step, infer_only=False):
        self.model.deal(step, infer_only=infer_only)

    def step_shares(self, Xs, Ys, step, deal=True):
        if deal:
            self.model.deal(step)
        self.model.train_step(Xs, Ys, step)

    def step(self, X, Y, step):
        Xs, Ys = self.share_batch(X, Y, step)
        self.step_shares(Xs, Ys, step)

    def step_dp(self, Xs, Ys, step, group=None, deal=True):
        """Data-parallel step: local forward/backward, all-reduce of gradient shares, update."""
        import torch.distributed as dist
        if deal:
            self.model.deal(step)
        self.model.forward_backward(Xs, Ys, step)
        world = dist.get_world_size(group) if dist.is_initialized() else 1
        ring_allreduce_(self.grad_tensor(), group)
        self.model.apply_update(extra_shift=self.update_shift(world))

    def update_shift(self, world):
        """Extra truncation of the summed gradient: log2(pairs) when each pair trains its own
        batch (weak scaling); 0 under strong scaling, where the sum IS the global-batch gradient."""
        if self.strong_pairs > 1:
            if world != self.strong_pairs:
                raise ValueError(f"strong scaling over {self.strong_pairs} pairs, all-reduce over {world}")
            return 0
        return dp_update_shift(world)

    def last_yhat(self):
        """Prediction shares of the last step as two uint64 views of model-owned memory."""
        a, b, n = self.model.output()
        return _wrap_device_ptr(a, n, "<u8"), _wrap_device_ptr(b, n, "<u8")

    def grad_tensor(self):
        """int64 view of the model-owned [2][P] gradient buffer (for the all-reduce)."""
        ptr, words = self.model.grads()
        return _wrap_device_ptr(ptr, 2 * words)

    def infer_shares(self, Xs, step):
        self.model.deal(step, infer_only=True)
        return self.model.infer(Xs, step, (Xs[0].shape[0], self.out_dim))

    # --- decode (client side, test/report only) ---------------------------------------------------
    def master_weights(self):
        out = []
        for layer in range(self.model.n_layers):
            W0, W1 = self.model.get_master(layer)
            out.append(psml.decode(self.master_ring, psml.reconstruct(self.ring, W0, W1)))
        return out

    def master_shares(self, layer):
        return self.model.get_master(layer)

    def close(self):
        self.model.close()
        self.ctx.close()


class PartyTrainer(SecureTrainer):
    """One party of the split deployment (Fig. 1b: the two servers in different
    processes / GPUs).  The party holds only its own shares; every opening of the step goes
    through `transport` (psml.Transport: peer memory over NVLink / CUDA IPC, NCCL, or a
    host-staged callback) and its untruncated gradient share is summed over its data-parallel
    group by the library-owned communicator `dp` (psml.DataParallel, None = one pair).
    The dealer runs in each party's process and each party reads only its own half of the
    material (the offline phase a deployment ships from the client)."""

    def __init__(self, task, W_init, party, transport, batch=128, pair_id=0, dp=None, w_share=None, **kw):
        """w_share: this party's master-weight shares (one tensor per layer) from the client; the
        model then never holds the peer's share (the peer slot is zero).  Without it the
        simulation shares W_init itself and then zeroes the peer's slot."""
        if w_share is not None:
            kw["w_shares"] = [(w, torch.zeros_like(w)) if party == 0 else (torch.zeros_like(w), w) for w in w_share]
        super().__init__(task, W_init, batch=batch, pair_id=pair_id, **kw)
        self.party = party
        self.xport = transport
        self.dp = dp
        if w_share is None:   # keep only this party's weight share
            for layer in range(self.model.n_layers):
                pair = list(self.model.get_master(layer))
                pair[1 - party].zero_()
                self.model.set_master(layer, tuple(pair))

    def share_batch(self, X, Y, step):
        """Client role: encode + share; this party receives only its own share."""
        Xs, Ys = super().share_batch(X, Y, step)
        return Xs[self.party], Ys[self.party]

    def step_party(self, X_i, Y_i, step, dp_group=None, dp_world=1, deal=True):
        """Forward/backward with per-round exchanges, all-reduce of this party's gradient share
        over the party's data-parallel group, update of this party's weights.  With a library
        communicator (self.dp) the whole step is one call (psml_party_train_step); a
        torch.distributed group (dp_group) is the host-side alternative."""
        if deal:
            self.model.deal(step)
        if self.dp is not None or dp_world == 1:
            self.model.party_train_step(self.party, self.xport, self.dp, X_i, Y_i, step)
            return
        self.model.party_forward_backward(self.party, self.xport, X_i, Y_i, step)
        ptr, words = self.model.grads()
        g = _wrap_device_ptr(ptr + 8 * words * self.party, words)
        ring_allreduce_(g, dp_group)
        self.model.party_apply_update(self.party, extra_shift=self.update_shift(dp_world))

    def capture_party(self, pipelined=True):
        """Capture this party's whole step (dealer [pipelined], online phase with its exchanges,
        gradient all-reduce, update) into CUDA graph(s) reading fixed share buffers."""
        d_in = self.d_in()
        self.Xi = torch.zeros((self.batch, d_in), dtype=torch.uint64, device="cuda")
        self.Yi = torch.zeros((self.batch, self.out_dim), dtype=torch.uint64, device="cuda")
        self.gstream = torch.cuda.Stream()
        self.gstream.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(self.gstream):
            self.model.party_capture_step(self.party, self.xport, self.dp, self.Xi, self.Yi, with_deal=True,
                                          with_update=True, pipelined=pipelined, stream=self.gstream)
        torch.cuda.current_stream().wait_stream(self.gstream)
        self.pipelined = pipelined
        self._next_dealt = None

    def graph_step_party(self, X_i, Y_i, step):
        """Copy this party's shares into the captured buffers and replay the captured step."""
        self.Xi.copy_(X_i.view(self.Xi.shape), non_blocking=True)
        self.Yi.copy_(Y_i.view(self.Yi.shape), non_blocking=True)
        if self.pipelined and self._next_dealt != step:
            self.model.deal(step)
        self.model.step_graph(step)
        self._next_dealt = step + 1

    def step(self, X, Y, step):
        X_i, Y_i = self.share_batch(X, Y, step)
        self.step_party(X_i, Y_i, step)

    def my_master_share(self, layer):
        return self.model.get_master(layer)[self.party]


def _dev64(X):
    """A contiguous float64 CUDA tensor of the plaintext batch (no copy if it already is one)."""
    t = torch.as_tensor(X, dtype=torch.float64)
    return (t if t.is_cuda else t.cuda()).contiguous()


def _wrap_device_ptr(ptr, numel, typestr="<i8"):
    """A torch tensor aliasing `numel` 8-byte words of library-owned device memory."""
    class _Holder:
        __cuda_array_interface__ = {"shape": (numel,), "typestr": typestr, "data": (ptr, False),
                                    "version": 3, "strides": None}
    return torch.as_tensor(_Holder(), device="cuda")
