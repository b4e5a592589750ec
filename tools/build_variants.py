"""Build tuning variants of libsr next to the product library (SR_LIB selects one)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cgo_damanijskymg20_b200 import build as B  # noqa: E402

VARIANTS = {
    "libsr_t640.so": ["SR_MCML_MAXT=640", "SR_MCML_MINB=2"],
    "libsr_t512.so": ["SR_MCML_MAXT=512", "SR_MCML_MINB=2"],
    "libsr_t576.so": ["SR_MCML_MAXT=576", "SR_MCML_MINB=2"],
    "libsr_t704.so": ["SR_MCML_MAXT=704", "SR_MCML_MINB=2"],
    "libsr_t448m3.so": ["SR_MCML_MAXT=448", "SR_MCML_MINB=3"],
    "libsr_t416m3.so": ["SR_MCML_MAXT=416", "SR_MCML_MINB=3"],
    "libsr_t768.so": ["SR_MCML_MAXT=768", "SR_MCML_MINB=2"],
    "libsr_t1024.so": ["SR_MCML_MAXT=1024", "SR_MCML_MINB=1"],
    "libsr_t384.so": ["SR_MCML_MAXT=384", "SR_MCML_MINB=3"],
    "libsr_t512m3.so": ["SR_MCML_MAXT=512", "SR_MCML_MINB=3"],
    "libsr_t480m3.so": ["SR_MCML_MAXT=480", "SR_MCML_MINB=3"],
    "libsr_pts5.so": ["SR_PT_MINB_SPEC=5"],
    "libsr_pts7.so": ["SR_PT_MINB_SPEC=7"],
    "libsr_ptp6.so": ["SR_PT_MINB_PDOM=6"],
    "libsr_ch16.so": ["SR_MC_CHUNK=16"],
    "libsr_ch32.so": ["SR_MC_CHUNK=32"],
    "libsr_ch128.so": ["SR_MC_CHUNK=128"],
    "libsr_pt9.so": ["SR_PT_MINB_SPEC=9", "SR_PT_MINB_PDOM=9"],
    "libsr_pt10.so": ["SR_PT_MINB_SPEC=10", "SR_PT_MINB_PDOM=10"],
    "libsr_pt8.so": ["SR_PT_MINB_SPEC=8", "SR_PT_MINB_PDOM=8"],
    "libsr_pt7.so": ["SR_PT_MINB_SPEC=7", "SR_PT_MINB_PDOM=7"],
    "libsr_ptbb.so": ["SR_PT_BOX_BRANCH"],
    "libsr_ptrows.so": ["SR_PT_ROWS"],
    "libsr_ptttb.so": ["SR_PT_TT_BRANCH"],
    "libsr_ptpp8.so": ["SR_PT_POOL_PAIRED", "SR_PT_MINB_SPEC=8"],
    "libsr_pts8.so": ["SR_PT_MINB_SPEC=8"],
    "libsr_ptpp.so": ["SR_PT_POOL_PAIRED"],
}
if __name__ == "__main__":
    names = sys.argv[1:] or list(VARIANTS)
    for n in names:
        print(B.build(force=True, defines=VARIANTS[n], lib=os.path.join(B.HERE, n)))
