"""Region file (FILE|lo|hi|name) for tools/ncu_regions.py / ncu_opmix2.py from the current
map.cu: the line span of each named device function, plus loops inside wc_window_tab."""
import re
import sys

src = open("paper_conf_ipps_jim11_b200/csrc/map.cu").read().split("\n")
names = ["word_mask4", "slow_word_len", "smem_word_at", "comb_add", "exact_key30_bf", "comb_or_table", "wc_drain",
         "wc_drain_tab", "wc_window_tab", "wc_window", "wc_map_loop", "flush_loop", "producer_loop", "finish_stage",
         "map_wait", "helper_wait", "ii_window", "ii_drain", "ii_map_loop", "reserve", "commit", "seal", "k_map"]
out = []
for n in names:
    for i, l in enumerate(src):
        if re.search(r"\b" + n + r"\(", l) and ("__device__" in l or "__global__" in l or
                                                 (i > 0 and ("template" in src[i - 1] or "__device__" in src[i - 1]))):
            if l.rstrip().endswith(";"):
                continue
            depth, j, started = 0, i, False
            while j < len(src):
                depth += src[j].count("{") - src[j].count("}")
                if "{" in src[j]:
                    started = True
                if started and depth <= 0:
                    break
                j += 1
            out.append((i + 1, j + 1, n))
            break
# sub-regions of wc_window_tab
for lo, hi, n in list(out):
    if n == "wc_window_tab":
        for k in range(lo, hi):
            if "for (uint32_t E = S & near" in src[k - 1]:
                e0 = k
            if "uint32_t L = S & ~near" in src[k - 1]:
                l0 = k
        out.remove((lo, hi, n))
        out += [(lo, e0 - 1, "tab classify"), (e0, l0 - 1, "tab exact loop"), (l0, hi, "tab long words")]
for lo, hi, n in sorted(out):
    print(f"map.cu|{lo}|{hi}|{n}")
print("common.cuh|1|80|common mbar")
print("common.cuh|81|400|common other")
print("kernels.h|1|400|kernels.h")
