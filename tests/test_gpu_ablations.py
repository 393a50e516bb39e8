"""Ablations of SURVEY §8(d) under the same parity contract (``-m gpu``): the paper's
segmented relaunch (ablation ii; Table IV) with several NumIteration[]
schedules must give the oracle's results bit for bit, like every other kernel."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import phantom
from tests.test_gpu_parity import _threads, assert_parity, gpu_run, pt, tracker  # noqa: F401

pytestmark = pytest.mark.gpu

REC = 1 | 2 | 4


@pytest.mark.parametrize("schedule", [(1,), (7,), "B", "C", (2000,)])
def test_segmented_relaunch_parity(pt, tracker, schedule):
    """A_1, A_7, strategy B, strategy C and a single segment (A_MaxStep) on a dispersed
    crossing: every particle's (nsteps, reason, end) and the map bit-exact."""
    sched = {"B": pt.SEGMENTS_B, "C": pt.SEGMENTS_C}.get(schedule, schedule)
    w = phantom.crossing(sigma=0.15, f_jitter=0.03, nseeds=200, particles_per_seed=300)
    tracker.set_segments(sched)
    g = gpu_run(tracker, w, REC | pt.PT_KERNEL_SEGMENTED)
    r = oracle.track(w, threads=_threads())
    assert_parity(g, r)
    assert g["stats"]["total_steps"] == int(r["nsteps"].sum())
    assert g["stats"]["particles"] == w.nparticles


def test_segmented_paper_mode_and_edges(pt, tracker):
    """Paper mode (NEXT-1), seeds outside the mask, max_steps reached inside a segment."""
    w = phantom.crossing(sigma=0.15, f_jitter=0.03, nseeds=50, particles_per_seed=64)
    seeds = w.seeds.copy()
    seeds[0] = (0.5, 0.5, 0.5)
    seeds[1] = (-3.0, 1.0, 1.0)
    tracker.set_segments(pt.SEGMENTS_B)
    for wv in (w.replace(seeds=seeds, sample_mode=1), w.replace(seeds=seeds, max_steps=37)):
        g = gpu_run(tracker, wv, REC | pt.PT_KERNEL_SEGMENTED)
        assert_parity(g, oracle.track(wv))
    for bad in (pt.PT_REC_PATHS, pt.PT_BIDIR, pt.PT_KERNEL_SIMPLE):
        with pytest.raises(pt.PtError) as e:
            tracker.track_workload(w, flags=pt.PT_KERNEL_SEGMENTED | bad, path_stride=4)
        assert e.value.status == pt.PT_ERR_ARG
    with pytest.raises(pt.PtError):
        tracker.set_segments([])
    with pytest.raises(pt.PtError):
        tracker.set_segments([5, 0])
