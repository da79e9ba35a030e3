"""Cross-process channel (one process per GPU).  The GPU cases run the worker
under torchrun with every rank on cuda:0 (CUDA-IPC to the same device): the
same registration / peer-mapping / notification / install code that spans
GPUs on an 8-GPU box.  The CPU case checks the bootstrap allgather marshalling
over a world-size-2 gloo group."""
import os
import socket
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def run_torchrun(nproc, script, args, timeout=240, env=None):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nproc}",
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()), script] + args
    e = dict(os.environ)
    e.update(env or {})
    r = subprocess.run(cmd, cwd=ROOT, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, timeout=timeout, text=True,
                       env=e)
    return r.returncode, r.stdout


@pytest.mark.gpu
@pytest.mark.parametrize("nproc,tier,mode,config", [
    (2, 0, 0, "ptychonn"), (4, 0, 0, "small"), (3, 0, 1, "small"), (2, 1, 0, "small"), (3, 1, 1, "ptychonn"),
])
def test_xproc_parity(nproc, tier, mode, config):
    rc, out = run_torchrun(nproc, "tests/xproc_worker.py",
                           ["--config", config, "--tier", str(tier), "--mode", str(mode)])
    assert rc == 0 and "XPROC_RESULT errors=0" in out, out[-4000:]


@pytest.mark.gpu
@pytest.mark.parametrize("nproc,mode,config", [(4, 0, "ptychonn"), (3, 0, "small"), (4, 1, "small"),
                                              (5, 0, "resnet50")])
def test_xproc_scatter_allgather(nproc, mode, config):
    rc, out = run_torchrun(nproc, "tests/xproc_worker.py",
                           ["--config", config, "--mode", str(mode), "--fanout", "2", "--versions", "5"])
    assert rc == 0 and "XPROC_RESULT errors=0" in out, out[-4000:]


@pytest.mark.gpu
@pytest.mark.parametrize("nproc,mode,fanout,no_peer_rank,expect", [
    (3, 0, 0, -1, 0), (3, 1, 0, -1, 0), (3, 0, 0, 2, 1), (2, 1, 0, 1, 1), (2, 0, 0, 0, 0),
    (4, 0, 2, -1, 0), (4, 0, 2, 3, 1), (3, 1, 1, 1, 1)])
def test_xproc_transfer_selector(nproc, mode, fanout, no_peer_rank, expect):
    """VIPER_TIER_AUTO (Transfer Selector): every rank resolves the
    same tier from the bootstrap's reachability round -- GPU while every consumer
    reaches the producer's GPU, DRAM as soon as one rank reports it cannot
    (VIPER_TEST_NO_PEER on that rank) -- and the updates stay bit-exact.  The
    producer's own reach does not matter: consumers pull from it."""
    rc, out = run_torchrun(nproc, "tests/xproc_worker.py",
                           ["--config", "small", "--tier", "2", "--mode", str(mode), "--versions", "4",
                            "--expect-tier", str(expect), "--no-peer-rank", str(no_peer_rank),
                            "--fanout", str(fanout)])
    assert rc == 0 and "XPROC_RESULT errors=0" in out, out[-4000:]


@pytest.mark.gpu
def test_xproc_scatter_allgather_fault():
    rc, out = run_torchrun(4, "tests/xproc_worker.py", ["--config", "small", "--fanout", "2", "--fault", "1",
                                                       "--versions", "3"])
    assert rc == 0 and "XPROC_RESULT errors=0" in out, out[-4000:]


@pytest.mark.gpu
@pytest.mark.parametrize("nproc,mode,config", [(3, 0, "ptychonn"), (4, 0, "small"), (4, 1, "small"),
                                              (5, 0, "resnet50")])
def test_xproc_chain(nproc, mode, config):
    """Pipelined chain fan-out (SURVEY s8(e) option 3): consumer i pulls every
    item from consumer i-1's staging, verifies it and stages it for i+1."""
    rc, out = run_torchrun(nproc, "tests/xproc_worker.py",
                           ["--config", config, "--mode", str(mode), "--fanout", "1", "--versions", "5"])
    assert rc == 0 and "XPROC_RESULT errors=0" in out, out[-4000:]


@pytest.mark.gpu
def test_xproc_chain_fault():
    """A flipped bit in one chain link's copy: that consumer reports
    VIPER_E_CHECKSUM and keeps serving the previous version (the worker checks
    it); its successor heals from the producer."""
    rc, out = run_torchrun(4, "tests/xproc_worker.py", ["--config", "small", "--fanout", "1", "--fault", "1",
                                                       "--versions", "3"])
    assert rc == 0 and "XPROC_RESULT errors=0" in out, out[-4000:]


@pytest.mark.gpu
@pytest.mark.parametrize("nproc,fanout,mode", [(2, 0, 0), (3, 0, 1), (4, 2, 0), (4, 1, 0), (3, 1, 1)])
def test_xproc_early_notify_pipeline(nproc, fanout, mode):
    """Cross-GPU item pipeline: v is published right after the pack launch and
    consumers' install kernels wait per item on seals released at system scope
    (forced on here, where all ranks share one GPU)."""
    rc, out = run_torchrun(nproc, "tests/xproc_worker.py",
                           ["--config", "resnet50", "--fanout", str(fanout), "--mode", str(mode), "--versions", "4"],
                           env={"VIPER_EARLY_NOTIFY": "1"})
    assert rc == 0 and "XPROC_RESULT errors=0" in out, out[-4000:]


@pytest.mark.gpu
def test_xproc_early_notify_waits_for_the_stream():
    """Early notification names v by a stream memop right before the pack: with
    300 ms of earlier work queued on the producer's stream, a consumer's install
    (launch -> done) stays short instead of spinning on its GPU for 300 ms."""
    rc, out = run_torchrun(2, "tests/xproc_worker.py",
                           ["--config", "resnet50", "--mode", "1", "--versions", "3", "--delay-ms", "300"],
                           env={"VIPER_EARLY_NOTIFY": "1"})
    assert rc == 0 and "XPROC_RESULT errors=0" in out, out[-4000:]


@pytest.mark.gpu
@pytest.mark.parametrize("nproc,fanout", [(3, 0), (4, 2), (4, 1)])
def test_xproc_no_torn_reads(nproc, fanout):
    rc, out = run_torchrun(nproc, "tests/xproc_worker.py", ["--config", "small", "--mode", "1", "--fanout",
                                                           str(fanout), "--stress", "1", "--versions", "200"])
    assert rc == 0 and "XPROC_RESULT errors=0" in out, out[-4000:]


@pytest.mark.gpu
@pytest.mark.parametrize("nproc,nprod,mode,config", [(3, 2, 0, "ptychonn"), (5, 2, 0, "resnet50"),
                                                    (5, 3, 1, "small"), (4, 2, 1, "ptychonn")])
def test_xproc_data_parallel_producers(nproc, nprod, mode, config):
    """data-parallel producers each pack their chunk share;
    consumers assemble every version from all of them."""
    rc, out = run_torchrun(nproc, "tests/xproc_worker.py", ["--config", config, "--mode", str(mode), "--nprod",
                                                           str(nprod), "--versions", "5"])
    assert rc == 0 and "XPROC_RESULT errors=0" in out, out[-4000:]


@pytest.mark.gpu
def test_xproc_consumer_process_death_is_detected():
    """A consumer process exits without unregistering: the SYNC producer notices
    (pid liveness in the shared control block) instead of stalling, and the
    surviving consumer keeps installing every version."""
    rc, out = run_torchrun(3, "tests/xproc_fail_worker.py", [], timeout=180)
    assert "FAIL_PRODUCER" in out and "ok=True" in out, out[-4000:]
    assert "FAIL_SURVIVOR version=6 good=True" in out, out[-4000:]


@pytest.mark.gpu
def test_xproc_fault_injection():
    rc, out = run_torchrun(3, "tests/xproc_worker.py", ["--config", "small", "--fault", "1", "--versions", "3"])
    assert rc == 0 and "XPROC_RESULT errors=0" in out, out[-4000:]


def test_bootstrap_allgather_gloo_world2():
    rc, out = run_torchrun(2, "tests/bootstrap_worker.py", [], timeout=120)
    assert rc == 0 and "BOOTSTRAP_OK" in out, out[-3000:]


def test_bootstrap_pre_failure_does_not_hang():
    """A rank failing before the bootstrap still joins its allgathers (CPU: both
    ranks fail with "no CUDA device"; GPU box: rank 1's host tensor is rejected
    and rank 0 gets VIPER_E_PEER)."""
    rc, out = run_torchrun(2, "tests/bootstrap_abort_worker.py", [], timeout=120)
    assert rc == 0 and "ABORT_OK" in out, out[-3000:]


@pytest.mark.gpu
def test_bootstrap_pre_failure_does_not_hang_gpu():
    """Same on a GPU box: rank 0 reaches the bootstrap and must fail with VIPER_E_PEER."""
    rc, out = run_torchrun(2, "tests/bootstrap_abort_worker.py", [], timeout=120)
    assert rc == 0 and "ABORT_OK" in out, out[-3000:]


def test_protocol_two_processes_gloo_cpu():
    """The cross-process version protocol on a real shm segment, CPU only:
    0 torn snapshot copies, 0 torn reads, no version regress over 3000 publishes."""
    rc, out = run_torchrun(2, "tests/protocol_worker.py", [], timeout=180)
    assert rc == 0 and "PROTO_RESULT errors=0" in out, out[-3000:]


@pytest.mark.gpu
@pytest.mark.parametrize("nproc,mode,config", [(2, 0, "ptychonn"), (3, 0, "small"), (4, 1, "small"),
                                              (2, 0, "resnet50"), (5, 0, "resnet50")])
def test_xproc_push(nproc, mode, config):
    """VIPER_FANOUT_PUSH: the producer's pack stores every item into
    each consumer's peer-mapped staging and releases its seal there; consumers
    install from local memory.  Bit-exact slots and installed-slot seals ==
    the oracle's, every version."""
    rc, out = run_torchrun(nproc, "tests/xproc_worker.py",
                           ["--config", config, "--mode", str(mode), "--fanout", "4", "--versions", "5"])
    assert rc == 0 and "XPROC_RESULT errors=0" in out, out[-4000:]


@pytest.mark.gpu
@pytest.mark.parametrize("nproc,fanout", [(3, 4), (2, 4)])
def test_xproc_push_early_notify(nproc, fanout):
    """Push with the cross-GPU item pipeline forced on: consumers wait per item
    on the seals the producer releases (system scope) into their staging."""
    rc, out = run_torchrun(nproc, "tests/xproc_worker.py",
                           ["--config", "resnet50", "--fanout", str(fanout), "--versions", "4"],
                           env={"VIPER_EARLY_NOTIFY": "1"})
    assert rc == 0 and "XPROC_RESULT errors=0" in out, out[-4000:]


@pytest.mark.gpu
@pytest.mark.parametrize("nproc,mode,config", [(2, 0, "ptychonn"), (3, 1, "small"), (3, 0, "resnet50")])
def test_xproc_copy_engine_fanout(nproc, mode, config):
    """VIPER_FANOUT_CE (SURVEY B2 as an engine mode): consumers copy the sealed
    snapshot with cudaMemcpyAsync, then install + verify locally."""
    rc, out = run_torchrun(nproc, "tests/xproc_worker.py",
                           ["--config", config, "--mode", str(mode), "--fanout", "101", "--versions", "4"])
    assert rc == 0 and "XPROC_RESULT errors=0" in out, out[-4000:]


@pytest.mark.gpu
def test_xproc_push_fault():
    rc, out = run_torchrun(3, "tests/xproc_worker.py", ["--config", "small", "--fanout", "4", "--fault", "1",
                                                       "--versions", "3"])
    assert rc == 0 and "XPROC_RESULT errors=0" in out, out[-4000:]


@pytest.mark.gpu
@pytest.mark.parametrize("nproc,mode", [(2, 0), (3, 0), (2, 1)])
def test_xproc_nccl_bit_exact_or_unsupported_everywhere(nproc, mode):
    """VIPER_FANOUT_NCCL (the NCCL-broadcast baseline inside the engine):
    bit-exact with one GPU per rank and SYNC; ranks sharing a GPU (NCCL refuses
    that) or an ASYNC producer give VIPER_E_UNSUPPORTED on every rank."""
    rc, out = run_torchrun(nproc, "tests/xproc_worker.py",
                           ["--config", "resnet50", "--fanout", "100", "--mode", str(mode), "--versions", "4",
                            "--allow-unsupported"])
    assert rc == 0, out[-4000:]
    assert "XPROC_RESULT errors=0" in out or "XPROC_UNSUPPORTED everywhere=True" in out, out[-4000:]
    if mode == 1:
        assert "XPROC_UNSUPPORTED everywhere=True" in out, out[-4000:]


@pytest.mark.gpu
@pytest.mark.parametrize("nproc", [2, 3])
def test_xproc_nvls_bit_exact_or_unsupported_everywhere(nproc):
    """VIPER_FANOUT_NVLS: bit-exact where the box exposes multicast (one GPU per
    rank, fabric manager); otherwise EVERY rank's registration fails with
    VIPER_E_UNSUPPORTED (a 1-GPU lease: ranks share a GPU) -- never a hang or a
    mixed outcome."""
    rc, out = run_torchrun(nproc, "tests/xproc_worker.py",
                           ["--config", "resnet50", "--fanout", "3", "--versions", "4", "--allow-unsupported"])
    assert rc == 0, out[-4000:]
    assert "XPROC_RESULT errors=0" in out or "XPROC_UNSUPPORTED everywhere=True" in out, out[-4000:]


@pytest.mark.gpu
def test_xproc_dram_install_does_not_hang_on_a_vanished_producer():
    """a DRAM-tier consumer whose producer named v but never raised
    the pieces' flags (VIPER_TEST_DRAM_STALL) gives the install up once the
    producer unregisters: VIPER_E_PEER, v not installed, prompt unregister."""
    rc, out = run_torchrun(2, "tests/xproc_stall_worker.py", [], timeout=120)
    assert "STALL_CONSUMER" in out and "ok=True" in out, out[-4000:]


def test_nvls_descriptor_handoff_gloo_cpu():
    """The NVLS registration's fd hand-off (abstract Unix socket + SCM_RIGHTS),
    CPU only: a served descriptor arrives in the other process and reads back
    the same bytes; a missing fetcher / server fails with VIPER_E_PEER in
    bounded time."""
    rc, out = run_torchrun(2, "tests/fdpass_worker.py", [], timeout=120)
    assert rc == 0 and "FDPASS rank0 ok=True" in out and "FDPASS rank1 ok=True" in out, out[-3000:]


@pytest.mark.gpu
@pytest.mark.parametrize("mode,early,config", [(0, "0", "resnet50"), (1, "0", "small"), (0, "1", "resnet50"),
                                              (1, "1", "ptychonn")])
def test_xproc_nvls_kernel_path_unicast(mode, early, config):
    """NVLS where the box has no multicast: VIPER_TEST_NVLS_UNICAST maps the
    "multicast" address to the one consumer's staging (CUDA IPC) and makes it
    the producer's snapshot, as its share of the object would be.  Runs
    pack_nvls_kernel (multimem.st -- on sm_100 the same global store) and the
    consumer's NVLS install path, with the early-notified item pipeline and
    without; bit-exact slots and installed-slot seals == the oracle's."""
    rc, out = run_torchrun(2, "tests/xproc_worker.py",
                           ["--config", config, "--mode", str(mode), "--fanout", "3", "--versions", "5"],
                           env={"VIPER_TEST_NVLS_UNICAST": "1", "VIPER_EARLY_NOTIFY": early})
    assert rc == 0 and "XPROC_RESULT errors=0" in out, out[-4000:]


@pytest.mark.gpu
@pytest.mark.parametrize("fanout", ["sa", "push", "nvls"])
def test_example_fanout_serve(fanout):
    """examples/fanout_serve.py: a trainer process publishes every step, two
    inference processes serve from the latest version and end with seals equal
    to the producer's and logits equal to the trainer's, bit for bit (NVLS falls
    back to direct pulls where multicast is unavailable)."""
    rc, out = run_torchrun(3, "examples/fanout_serve.py", ["--fanout", fanout, "--steps", "20"], timeout=300)
    assert rc == 0 and f"FANOUT_SERVE ok ({fanout})" in out, out[-4000:]
