"""Write workloads/shapes.json: the per-tensor parameter counts of the models whose
gradients the synthetic workloads mimic (Table 2(b)).
Built on device="meta" (no weights, no network). ResNet-20 (CIFAR, option-A shortcuts)
is built from its formula."""
import json, torch, torchvision
from transformers import BertConfig, BertModel, GPT2Config, GPT2LMHeadModel

def sizes(m):
    return [int(p.numel()) for _, p in m.named_parameters()]

def resnet20():
    out = [16 * 3 * 9, 16, 16]                       # conv1 + bn1
    cin = 16
    for cout in (16, 32, 64):
        for b in range(3):
            out += [cout * cin * 9, cout, cout, cout * cout * 9, cout, cout]
            cin = cout
    out += [10 * 64, 10]                             # fc
    return out

shapes = {}
shapes["resnet20"] = resnet20()
with torch.device("meta"):
    shapes["resnet50"] = sizes(torchvision.models.resnet50())
    shapes["vgg16"] = sizes(torchvision.models.vgg16())
    shapes["bert_large"] = sizes(BertModel(BertConfig(hidden_size=1024, num_hidden_layers=24,
                                                      num_attention_heads=16, intermediate_size=4096)))
    shapes["gpt2_xl"] = sizes(GPT2LMHeadModel(GPT2Config(n_embd=1600, n_layer=48, n_head=25)))
for k, v in shapes.items():
    print(k, len(v), sum(v))
json.dump(shapes, open("workloads/shapes.json", "w"))
