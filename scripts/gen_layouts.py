"""Regenerate the synthetic bucket layouts of SURVEY.md Appendix A.

Parameter shapes come from torchvision ResNet-50 / VGG-19 / Swin-B and
transformers BertForQuestionAnswering (BERT-base, the SQuAD QA head of the
paper's Table 1).  Buckets follow DDP's default
assignment (reverse registration order, 1 MiB first bucket then 25 MiB),
the bucketing the paper's D1 persists.

Writes paper_conf_sc_lixyszrljlllq23_b200/layouts.json:
  {model: {"dtype": "f32"|"bf16", "buckets": [[tensor numel, ...], ...],
           "tensor_names": [[...], ...]}}
Only element counts are used downstream; no weights are loaded.
"""
import json
import os

import torch
import torch.distributed as dist


def _params(model):
    return [(n, p) for n, p in model.named_parameters() if p.requires_grad]


def _buckets(named, dtype):
    names = [n for n, _ in named][::-1]
    tensors = [torch.empty(p.numel(), dtype=dtype, device="meta") for _, p in named][::-1]
    # DDP: reversed registration order, caps [1 MiB, 25 MiB]
    idx_lists, _ = dist._compute_bucket_assignment_by_size(
        [torch.empty(t.numel(), dtype=dtype) for t in tensors], [1 << 20, 25 << 20])
    out, out_names = [], []
    for idxs in idx_lists:
        out.append([int(tensors[i].numel()) for i in idxs])
        out_names.append([names[i] for i in idxs])
    return out, out_names


def main():
    import torchvision
    import transformers

    models = {}
    with torch.device("meta"):
        r50 = torchvision.models.resnet50()
        vgg = torchvision.models.vgg19()
        swin = torchvision.models.swin_b()
        bert = transformers.BertForQuestionAnswering(transformers.BertConfig())
    for name, m, dt, tdt in [("resnet50", r50, "f32", torch.float32),
                              ("vgg19", vgg, "f32", torch.float32),
                              ("bert_base", bert, "bf16", torch.bfloat16),
                              ("swin_b", swin, "f32", torch.float32)]:
        b, n = _buckets(_params(m), tdt)
        models[name] = {"dtype": dt, "buckets": b, "tensor_names": n}
        print(name, [sum(x) for x in b], sum(sum(x) for x in b))
    # BN buffers of ResNet-50 (running_mean/var fp32 + num_batches_tracked int64)
    bn = [(n, tuple(t.shape), str(t.dtype)) for n, t in r50.named_buffers()]
    models["resnet50"]["bn_buffers"] = {
        "f32_numel": sum(int(torch.Size(s).numel()) for n, s, d in bn if d == "torch.float32"),
        "i64_count": sum(1 for n, s, d in bn if d == "torch.int64"),
        "n_layers": sum(1 for n, s, d in bn if n.endswith("running_mean")),
    }
    path = os.path.join(os.path.dirname(__file__), "..", "paper_conf_sc_lixyszrljlllq23_b200", "layouts.json")
    with open(path, "w") as f:
        json.dump(models, f)
    print(models["resnet50"]["bn_buffers"])


if __name__ == "__main__":
    main()
