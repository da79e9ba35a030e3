"""Train-and-serve with viper: a training loop publishes its weights every few
steps (ASYNC: the trainer only pays for the snapshot), while an
inference thread keeps serving from the latest installed version without ever
seeing a torn model (double buffer + atomic swap).

    python examples/train_and_serve.py [--steps 60] [--every 5]

At the end the served logits for a probe batch are compared with the
trainer's own logits at the same version (bitwise, same kernels)."""
import argparse
import os
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import torchvision
from torch.func import functional_call

from paper_conf_icpp_yecrbypnmskn24_b200 import viper as V


def main(steps=60, every=5, verbose=True):
    torch.manual_seed(0)
    dev = torch.device("cuda", 0)
    trainer = torchvision.models.resnet18(num_classes=10).to(dev)
    server = torchvision.models.resnet18(num_classes=10).to(dev).eval()
    # the whole state dict travels: parameters ("weights, biases")
    # and the buffers inference needs (BatchNorm running statistics); dtypes
    # are opaque to the path (num_batches_tracked is int64 bytes)
    names = list(trainer.state_dict().keys())
    prod = V.Model("resnet18", V.PRODUCER, list(trainer.state_dict().values()), mode=V.ASYNC, names=names)
    cons = V.Model("resnet18", V.CONSUMER, list(server.state_dict().values()), names=names)
    like = list(server.state_dict().values())
    opt = torch.optim.SGD(trainer.parameters(), lr=0.05, momentum=0.9)
    probe = torch.randn(8, 3, 64, 64, device=dev)
    stop = threading.Event()
    served = {"n": 0, "versions": set()}

    def serve():
        s = torch.cuda.Stream(device=dev)
        with torch.cuda.stream(s), torch.no_grad():
            while not stop.is_set():
                try:
                    view = cons.acquire_latest(timeout_us=100_000)
                except V.ViperError:
                    continue
                params = dict(zip(names, view.tensors(like)))
                functional_call(server, params, (probe,))
                cons.release(view, stream=s)  # unpinned once this stream ran the forward
                served["n"] += 1
                served["versions"].add(view.version)

    th = threading.Thread(target=serve)
    th.start()
    version = 0
    t0 = time.time()
    for step in range(1, steps + 1):
        x = torch.randn(32, 3, 64, 64, device=dev)
        y = torch.randint(0, 10, (32,), device=dev)
        loss = torch.nn.functional.cross_entropy(trainer(x), y)
        opt.zero_grad(set_to_none=False)
        loss.backward()
        opt.step()
        if step % every == 0:
            version += 1
            prod.publish(version, stream=torch.cuda.current_stream())  # snapshot after the optimizer step
            if verbose:
                print(f"step {step:4d} loss {loss.item():.4f} published v{version}", flush=True)
    cons.wait_installed(version, timeout_us=10_000_000)
    stop.set()
    th.join()
    # the served model at `version` == the trainer's weights at `version`
    trainer.eval()
    server.eval()
    with torch.no_grad():
        ref = trainer(probe)
        view = cons.acquire_latest()
        out = functional_call(server, dict(zip(names, view.tensors(like))), (probe,))
        cons.release(view)
    same = torch.equal(ref, out)
    if verbose:
        print(f"{steps} steps in {time.time() - t0:.2f}s; served {served['n']} requests on "
              f"{len(served['versions'])} versions; final logits identical: {same}", flush=True)
    cons.close()
    prod.close()
    return same, served


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=60)
    ap.add_argument("--every", type=int, default=5)
    a = ap.parse_args()
    ok, _ = main(a.steps, a.every)
    sys.exit(0 if ok else 1)
