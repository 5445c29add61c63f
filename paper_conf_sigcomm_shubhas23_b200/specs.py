"""Model architectures on the hot path, as plain op lists (no arithmetic here).

Each spec is ``{"name", "in_h", "in_w", "in_c", "ops": [...]}`` with ops
``conv(kh,kw,stride,pad,cout,act,residual)``, ``maxpool(k,stride,pad)``, ``block(cout,stride)``
(cout>0 -> 1x1 projection shortcut), ``exit(num_classes, loss_weight)``, ``det_head(...)``.
The same description is marshalled into the C-ABI's ``adainf_op`` (``binding.py``) and, by the tests
only, into the oracle's own ``or_op``.

Readings: exits at ResNet stage boundaries (Q3, "every 3 layers"),
GAP->FC exit heads (Q4), BN folded (Q10), TinyYOLOv3-like single-scale detector (Q18),
synthetic audio DAG (Q24).
"""
from __future__ import annotations

RELU, LEAKY, NONE, RELU6 = 1, 2, 0, 3

# TinyYOLOv3 13x13-scale anchors (w, h) in pixels (reading Q18)
YOLO_ANCHORS = [81.0, 82.0, 135.0, 169.0, 344.0, 319.0]


def conv(k, cout, stride=1, pad=None, act=RELU, residual=False, groups=1):
    """groups > 1: grouped conv (groups == cin == cout: depthwise, MobileNetV2 / ShuffleNet, NEXT-3);
    residual: True / 1 add the open block's shortcut, 2 concatenate it in front of this conv's channels"""
    return {"kind": "conv", "kh": k, "kw": k, "stride": stride, "pad": (k // 2) if pad is None else pad,
            "cout": cout, "act": act, "residual": int(residual), "groups": groups}


SHUFFLE_G8_STAGES = [(384, 4), (768, 8), (1536, 4)]  # ShuffleNet 1x, g = 8: (output channels, units) per stage


def shufflenet_ee(num_classes=10, in_hw=224, in_c=3, groups=8, width=1.0, exits_after=(0, 1)):
    """ShuffleNet (v1) early-exit classifier (the paper's video-DAG classifier family; NEXT-3): 3x3/2 conv 24
    + 3x3/2 max-pool, then per stage one stride-2 unit (3x3/2 average-pool shortcut concatenated with the branch)
    and stride-1 units (identity shortcut added); a unit = grouped 1x1 conv (bottleneck = out/4, ReLU; the first
    one of stage 2 dense) -> channel shuffle (g) -> 3x3 depthwise (stride, no act) -> grouped 1x1 conv (no act
    before the join) -> ReLU after the add / concat.  Exits after the stages in exits_after + the final exit
    (reading Q3)."""
    def ch(c):
        return max(8 * groups, int(round(c * width / (8 * groups))) * 8 * groups)
    ops = [conv(3, 24, stride=2), maxpool(3, 2, 1)]
    cin = 24
    for si, (cout, n) in enumerate(SHUFFLE_G8_STAGES):
        cout = ch(cout)
        for u in range(n):
            mid = cout // 4
            g1 = 1 if (si == 0 and u == 0) else groups
            if u == 0:
                ops += [block(stride=2, pool=1), conv(1, mid, groups=g1), shuffle(groups),
                        conv(3, mid, stride=2, act=NONE, groups=mid), conv(1, cout - cin, act=RELU, groups=groups,
                                                                       residual=2)]
            else:
                ops += [block(0), conv(1, mid, groups=groups), shuffle(groups), conv(3, mid, act=NONE, groups=mid),
                        conv(1, cout, act=RELU, groups=groups, residual=True)]
            cin = cout
        if si in exits_after:
            ops.append(exit_(num_classes))
    ops.append(exit_(num_classes))
    return {"name": "shufflenet_ee", "in_h": in_hw, "in_w": in_hw, "in_c": in_c, "ops": ops}


def maxpool(k, stride, pad=0):
    return {"kind": "maxpool", "kh": k, "kw": k, "stride": stride, "pad": pad}


def block(cout=0, stride=1, pool=0, k=3, pad=1):
    """cout > 0: 1x1 projection shortcut; pool = 1: k x k average-pool shortcut (stride, pad; zero padding counted,
    ShuffleNet stride-2 unit); else identity"""
    if pool:
        return {"kind": "block", "cout": 0, "stride": stride, "pool": 1, "kh": k, "kw": k, "pad": pad}
    return {"kind": "block", "cout": cout, "stride": stride}


def upsample(factor=2):
    """nearest-neighbour upsampling (TinyYOLOv3's second scale)"""
    return {"kind": "upsample", "stride": factor}


def route(a, b=-1):
    """current tensor := output of op a (absolute op index), concatenated with op b's along channels if b >= 0"""
    return {"kind": "route", "kh": a, "kw": b}


def shuffle(groups):
    """ShuffleNet channel shuffle (view (g, C/g) -> transpose -> flatten)"""
    return {"kind": "shuffle", "groups": groups}


def exit_(num_classes, loss_weight=1.0):
    return {"kind": "exit", "num_classes": num_classes, "loss_weight": loss_weight}


def tiny_cnn_ee(num_classes=10):
    """BASELINE config 1: 3-conv early-exit CNN, 2 exits, 32x32x3 (95,188 params)."""
    ops = [conv(3, 32), maxpool(2, 2), conv(3, 64), maxpool(2, 2), exit_(num_classes), conv(3, 128),
           exit_(num_classes)]
    return {"name": "tiny_cnn_ee", "in_h": 32, "in_w": 32, "in_c": 3, "ops": ops}


def _basic_block(cout, stride, cin):
    proj = stride != 1 or cin != cout
    return [block(cout if proj else 0, stride), conv(3, cout, stride=stride), conv(3, cout, residual=True)]


def resnet18_ee(num_classes=10, in_hw=224, in_c=3):
    """BASELINE config 2: ResNet-18 with exits after layer1..layer3 + final (11,181,352 params at 10 cls)."""
    ops = [conv(7, 64, stride=2, pad=3), maxpool(3, 2, 1)]
    cin = 64
    for cout, stride in ((64, 1), (128, 2), (256, 2), (512, 2)):
        ops += _basic_block(cout, stride, cin)
        ops += _basic_block(cout, 1, cout)
        ops.append(exit_(num_classes))
        cin = cout
    return {"name": "resnet18_ee", "in_h": in_hw, "in_w": in_hw, "in_c": in_c, "ops": ops}


def _inverted_residual(cin, cout, stride, t):
    """MobileNetV2 inverted residual (NEXT-3): 1x1 expand (ReLU6, skipped when t == 1) -> 3x3 depthwise
    (ReLU6) -> 1x1 linear projection, + identity shortcut when stride 1 and cin == cout."""
    hid = cin * t
    ops = []
    res = stride == 1 and cin == cout
    if res:
        ops.append(block(0))
    if t != 1:
        ops.append(conv(1, hid, act=RELU6))
    ops.append(conv(3, hid, stride=stride, act=RELU6, groups=hid))
    ops.append(conv(1, cout, act=NONE, residual=res))
    return ops


MNV2_STAGES = [(1, 16, 1, 1), (6, 24, 2, 2), (6, 32, 3, 2), (6, 64, 4, 2), (6, 96, 3, 1), (6, 160, 3, 2),
               (6, 320, 1, 1)]


def mobilenetv2_ee(num_classes=10, in_hw=224, in_c=3, width=1.0, exits_after=(1, 2, 4)):
    """MobileNetV2 early-exit classifier (the paper's video-DAG classifier; NEXT-3): stem 3x3/2 conv 32
    (ReLU6), inverted-residual stages (t, c, n, s) as in MobileNetV2, 1x1 conv 1280 (ReLU6); exits after the
    stages listed in exits_after (stage indices into MNV2_STAGES: 24-ch 56x56, 32-ch 28x28, 96-ch 14x14 at 224)
    + the final GAP -> FC head (reading Q3: exits at stage boundaries)."""
    def ch(c):
        return max(8, int(round(c * width / 8)) * 8)
    ops = [conv(3, ch(32), stride=2, act=RELU6)]
    cin = ch(32)
    for si, (t, c, n, s_) in enumerate(MNV2_STAGES):
        for b in range(n):
            ops += _inverted_residual(cin, ch(c), s_ if b == 0 else 1, t)
            cin = ch(c)
        if si in exits_after:
            ops.append(exit_(num_classes))
    ops += [conv(1, ch(1280), act=RELU6), exit_(num_classes)]
    return {"name": "mobilenetv2_ee", "in_h": in_hw, "in_w": in_hw, "in_c": in_c, "ops": ops}


def tiny_yolo_det(in_hw=416, det_classes=2, anchors=3, width=512, nms_iou=0.0):
    """BASELINE config 3 detector: TinyYOLOv3-like single-scale, 'compressed' (layer 7 1024->512); nms_iou > 0
    adds greedy per-(frame, class) NMS before routing (NEXT-3, reading Q18b; TinyYOLOv3 uses 0.45)."""
    ops = []
    for c in (16, 32, 64, 128, 256):
        ops += [conv(3, c, act=LEAKY), maxpool(2, 2)]
    ops += [conv(3, 512, act=LEAKY), maxpool(3, 1, 1), conv(3, width, act=LEAKY), conv(1, 256, act=LEAKY),
            conv(3, 512, act=LEAKY), conv(1, anchors * (5 + det_classes), act=NONE),
            {"kind": "det_head", "anchors": anchors, "det_classes": det_classes, "grid_stride": 32,
             "anchor_wh": YOLO_ANCHORS[:2 * anchors], "nms_iou": nms_iou}]
    return {"name": "tiny_yolo_det", "in_h": in_hw, "in_w": in_hw, "in_c": 3, "ops": ops}


def _walk(spec):
    """(op index, op, H, W, C of the tensor entering the op, H, W, C after it) along the op list; BLOCK reports its
    shortcut's shape as the output.  A CONV with residual 2 concatenates the open block's shortcut channels."""
    H, W, Cc = spec["in_h"], spec["in_w"], spec["in_c"]
    blocks = []
    after = []  # the current tensor after each op (ROUTE sources)
    for i, o in enumerate(spec["ops"]):
        k = o["kind"]
        if k == "conv":
            Ho = (H + 2 * o["pad"] - o["kh"]) // o["stride"] + 1
            Wo = (W + 2 * o["pad"] - o["kw"]) // o["stride"] + 1
            Co = o["cout"]
            if o.get("residual", 0):
                sc = blocks.pop()
                if o["residual"] == 2:
                    Co += sc
            yield i, o, H, W, Cc, Ho, Wo, Co
            H, W, Cc = Ho, Wo, Co
        elif k == "maxpool":
            Ho = (H + 2 * o["pad"] - o["kh"]) // o["stride"] + 1
            Wo = (W + 2 * o["pad"] - o["kw"]) // o["stride"] + 1
            yield i, o, H, W, Cc, Ho, Wo, Cc
            H, W = Ho, Wo
        elif k == "upsample":
            yield i, o, H, W, Cc, H * o["stride"], W * o["stride"], Cc
            H, W = H * o["stride"], W * o["stride"]
        elif k == "route":
            Ho, Wo, Co = after[o["kh"]]
            if o.get("kw", -1) >= 0:
                Co += after[o["kw"]][2]
            yield i, o, H, W, Cc, Ho, Wo, Co
            H, W, Cc = Ho, Wo, Co
        elif k == "block":
            if o["cout"] > 0:
                Ho, Wo, Co = (H - 1) // o["stride"] + 1, (W - 1) // o["stride"] + 1, o["cout"]
            elif o.get("pool", 0):
                Ho = (H + 2 * o["pad"] - o["kh"]) // o["stride"] + 1
                Wo = (W + 2 * o["pad"] - o["kw"]) // o["stride"] + 1
                Co = Cc
            else:
                Ho, Wo, Co = H, W, Cc
            blocks.append(Co)
            yield i, o, H, W, Cc, Ho, Wo, Co
        else:
            yield i, o, H, W, Cc, H, W, Cc
        after.append((H, W, Cc))


YOLO_ANCHORS_26 = [10.0, 14.0, 23.0, 27.0, 37.0, 58.0]  # TinyYOLOv3's 26x26-scale anchors (w, h), pixels


def tiny_yolo_det2(in_hw=416, det_classes=2, anchors=3, width=512, nms_iou=0.45):
    """Two-scale TinyYOLOv3-like detector (NEXT-3, reading Q18c): the single-scale network (13x13 head, stride 32)
    plus TinyYOLOv3's second branch -- route from the 13x13 1x1-256 conv, 1x1 conv 128, x2 nearest upsample, concat
    with the 26x26x256 conv output, 3x3 conv 256, 1x1 head at stride 16 with the 26x26 anchors; detections of both
    scales merged in candidate order and NMS'd together per (frame, class)."""
    base = tiny_yolo_det(in_hw=in_hw, det_classes=det_classes, anchors=anchors, width=width, nms_iou=nms_iou)
    ops = list(base["ops"])
    ch = anchors * (5 + det_classes)
    assert ops[8]["kind"] == "conv" and ops[13]["kind"] == "conv" and ops[13]["kh"] == 1
    ops += [route(13), conv(1, 128, act=LEAKY), upsample(2), route(19, 8), conv(3, 256, act=LEAKY),
            conv(1, ch, act=NONE),
            {"kind": "det_head", "anchors": anchors, "det_classes": det_classes, "grid_stride": 16,
             "anchor_wh": YOLO_ANCHORS_26[:2 * anchors], "nms_iou": nms_iou}]
    return {"name": "tiny_yolo_det2", "in_h": in_hw, "in_w": in_hw, "in_c": 3, "ops": ops}


def num_params(spec) -> int:
    """Parameter count from the documented flat layout (include/adainf.h)."""
    return sum(int(__import__("math").prod(shp)) for _k, _i, _o, shp in param_segments(spec))


def param_segments(spec):
    """[(kind, op_index, offset, shape)] of the flat fp32 parameter vector, in layout order."""
    segs, off = [], 0
    for i, o, _H, _W, Cc, _Ho, _Wo, _Co in _walk(spec):
        k = o["kind"]
        if k == "conv":
            shp = (o["cout"], o["kh"], o["kw"], Cc // o.get("groups", 1))
            segs.append(("conv_w", i, off, shp))
            off += o["cout"] * o["kh"] * o["kw"] * (Cc // o.get("groups", 1))
            segs.append(("conv_b", i, off, (o["cout"],)))
            off += o["cout"]
        elif k == "block" and o["cout"] > 0:
            segs.append(("proj_w", i, off, (o["cout"], 1, 1, Cc)))
            off += o["cout"] * Cc
            segs.append(("proj_b", i, off, (o["cout"],)))
            off += o["cout"]
        elif k == "exit":
            segs.append(("exit_w", i, off, (Cc, o["num_classes"])))
            off += Cc * o["num_classes"]
            segs.append(("exit_b", i, off, (o["num_classes"],)))
            off += o["num_classes"]
    return segs


def macs_per_sample(spec):
    """Per-op forward MACs of one sample (conv + projection + exit FC), list aligned with ops."""
    out = []
    for _i, o, _H, _W, Cc, Ho, Wo, _Co in _walk(spec):
        k = o["kind"]
        m = 0
        if k == "conv":
            m = Ho * Wo * o["cout"] * o["kh"] * o["kw"] * (Cc // o.get("groups", 1))
        elif k == "block" and o["cout"] > 0:
            m = Ho * Wo * o["cout"] * Cc
        elif k == "exit":
            m = Cc * o["num_classes"]
        out.append(m)
    return out
