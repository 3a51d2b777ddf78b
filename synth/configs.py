"""The BASELINE.json workload configs as seeded synthetic recipes (INPUT GENERATION ONLY).

configs[0] tiny, [1] state-scale, [2] CONUS-scale (the bench workload at N=1), [3] CONUS
sharded by tile rows, [4] PIP-stress (50k jagged polygons, tile sweep 64..1024).
Recipes and seeds: SURVEY.md §8d, DESIGN.md "Input recipe".
"""
from __future__ import annotations

from dataclasses import dataclass, field

from .dem import NODATA, DemSpec
from .polygons import Polygons, conus_mask, voronoi_tiling

ARCSEC = 1.0 / 3600.0


@dataclass(frozen=True)
class Config:
    name: str
    rows: int
    cols: int
    gt: tuple
    dem: DemSpec
    n_seeds: int
    level: int
    poly_seed: int
    n_holes: int
    tile: int
    nbins: int
    lo: int = 0
    width: int = 1
    nodata: int | None = NODATA
    oor_drop: bool = False
    mask: str | None = None
    east_bias: float = 0.0
    extra: dict = field(default_factory=dict)

    @property
    def cells(self) -> int:
        return self.rows * self.cols

    def polygons(self) -> Polygons:
        m = conus_mask if self.mask == "conus" else None
        return voronoi_tiling(self.cols, self.rows, self.gt, self.n_seeds, self.level, self.poly_seed,
                              n_holes=self.n_holes, mask=m, east_bias=self.east_bias)

    def describe(self) -> dict:
        return {"workload": self.name, "rows": self.rows, "cols": self.cols, "cells": self.cells,
                "tile": self.tile, "nbins": self.nbins, "dem_seed": self.dem.seed,
                "poly_seed": self.poly_seed, "n_seeds": self.n_seeds, "jag_level": self.level}


TINY = Config("tiny", 1024, 1024, (0.0, 1.0, 0.0, 1024.0, 0.0, -1.0),
              DemSpec(seed=1, base=-150, macro_amp=900, fine_amp=200, void_thresh=12500),
              n_seeds=15, level=4, poly_seed=2, n_holes=1, tile=128, nbins=256)

# lon/lat-like variant of tiny (non-dyadic cell size), same cells
TINY_LONLAT = Config("tiny-lonlat", 1024, 1024, (-100.0, ARCSEC, 0.0, 40.0, 0.0, -ARCSEC),
                     DemSpec(seed=11, base=-150, macro_amp=900, fine_amp=200, void_thresh=12500),
                     n_seeds=15, level=4, poly_seed=12, n_holes=1, tile=128, nbins=256)

STATE = Config("state", 40000, 40000, (-106.0, ARCSEC, 0.0, 37.0, 0.0, -ARCSEC), DemSpec(seed=3),
               n_seeds=100, level=8, poly_seed=4, n_holes=3, tile=256, nbins=5000)

CONUS = Config("conus", 93600, 216000, (-126.0, ARCSEC, 0.0, 50.0, 0.0, -ARCSEC), DemSpec(seed=5),
               n_seeds=4560, level=9, poly_seed=6, n_holes=40, tile=256, nbins=5000, mask="conus",
               east_bias=0.3)

PIPSTRESS = Config("pip-stress", 93600, 216000, (-126.0, ARCSEC, 0.0, 50.0, 0.0, -ARCSEC), DemSpec(seed=5),
                   n_seeds=73500, level=7, poly_seed=7, n_holes=200, tile=256, nbins=5000, mask="conus")

CONFIGS = {c.name: c for c in (TINY, TINY_LONLAT, STATE, CONUS, PIPSTRESS)}
